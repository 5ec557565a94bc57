python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | tail -3
timeout 1500 python bench.py --config c5 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c5.json 2> gpurun_out/bench_c5.err
python -c "import json; d=json.load(open('gpurun_out/bench_c5.json')); print('c5', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, 'frac', round(d['roofline']['frac'],3), d['index']['last_scan'])" || tail -20 gpurun_out/bench_c5.err
grep "\[bench\]" gpurun_out/bench_c5.err | tail -3
timeout 600 python bench.py --config c2 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c2.json 2> gpurun_out/bench_c2.err
python -c "import json; d=json.load(open('gpurun_out/bench_c2.json')); print('c2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, 'frac', round(d['roofline']['frac'],3), d['index']['last_scan'])" || tail -5 gpurun_out/bench_c2.err
