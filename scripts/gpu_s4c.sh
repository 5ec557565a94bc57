# session-4: large-k select staging by cp.async + register-blocked bitonic sort
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/s4c
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -k "large_k or merge or edge or c1" 2>&1 | tail -2
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/s4c/b_$2_$3.json 2> gpurun_out/s4c/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/s4c/b_$2_$3.json')); print('$1 $2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, round(d['roofline']['frac'],3))" || tail -3 gpurun_out/s4c/b_$2_$3.err
}
run MV_NEED=0 c4 x
run MV_NEED=8192 c4 n8k
