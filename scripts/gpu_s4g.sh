# session-4: SQ8 item width by expected queries per list (4/8 TMEM accumulators), sample rows per list rule
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/s4g
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 2>&1 | tail -3
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/s4g/b_$2_$3.json 2> gpurun_out/s4g/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/s4g/b_$2_$3.json')); print('$1 $2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, round(d['roofline']['frac'],3))" || tail -3 gpurun_out/s4g/b_$2_$3.err
}
run MV_X=0 c5 x
run MV_SQ8_QC=16 c5 q16
run MV_SQ8_QC=64 c5 q64
run MV_X=0 c3 x
run MV_SQ8_QC=32 c3 q32
run MV_X=0 c4 x
run MV_X=0 c2 x
