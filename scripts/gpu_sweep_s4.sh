# session-4 sweep: the seeding bound's sample size (MV_NEED candidates, MV_CAPA rows per list)
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/w4
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -k "large_k" 2>&1 | tail -2
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/w4/b_$2_$3.json 2> gpurun_out/w4/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/w4/b_$2_$3.json')); print('$1 $2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()})" || tail -3 gpurun_out/w4/b_$2_$3.err
}
run MV_NEED=0 c4 base
run MV_NEED=8192 c4 n8k
run "MV_NEED=8192 MV_CAPA=1024" c4 n8kc1k
run MV_NEED=16384 c4 n16k
run MV_NEED=0 c3 base
run MV_NEED=400 c3 n400
run MV_NEED=800 c3 n800
run MV_NEED=1600 c3 n1600
run "MV_NEED=1600 MV_CAPA=256" c3 n1600c256
run MV_NEED=3200 c3 n3200
run "MV_NEED=3200 MV_CAPA=256" c3 n3200c256
run MV_NEED=40 c2 n40
run MV_NEED=80 c2 n80
run MV_NEED=160 c2 n160
run MV_NEED=0 c5 base
run MV_NEED=80 c5 n80
run MV_NEED=320 c5 n320
