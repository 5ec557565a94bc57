# session-4 sweep 2 (sparse emission path built in): seeding sample size around sqrt(k * candidates)
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/w5
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 2>&1 | tail -2
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/w5/b_$2_$3.json 2> gpurun_out/w5/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/w5/b_$2_$3.json')); print('$1 $2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()})" || tail -3 gpurun_out/w5/b_$2_$3.err
}
run MV_NEED=0 c2 base
run MV_NEED=100 c2 n100
run MV_NEED=0 c3 base
run MV_NEED=1100 c3 n1100
run MV_NEED=12288 c4 n12k
run MV_NEED=24576 c4 n24k
run MV_NEED=1000 c5 n1000
run MV_NEED=2000 c5 n2000
run MV_NEED=4000 c5 n4000
