python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | tail -15
for c in c2 c4; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
  python -c "import json; d=json.load(open('gpurun_out/bench_$c.json')); print('$c', round(d['value']), 'qps', d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, 'frac', round(d['roofline']['frac'],3), d['index']['last_scan'])" || tail -5 gpurun_out/bench_$c.err
done
