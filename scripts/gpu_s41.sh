python -c "import __graft_entry__ as g; g.build()" || exit 1
run() {
  env $1 timeout 1500 python bench.py --config ${2:-c2} --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$2.json 2> gpurun_out/bench_$2.err
  python -c "import json; d=json.load(open('gpurun_out/bench_$2.json')); print('$1 ${2:-c2}', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, 'frac', round(d['roofline']['frac'],3), d['index']['last_scan'])" || tail -3 gpurun_out/bench_$2.err
}
run MV_CAPA=128 c2
run MV_CAPA=160 c2
run MV_CAPA=64 c2
