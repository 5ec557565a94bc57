# session-4 final lines (sample rows-per-list rule): GPU tests, c2 default line with the CPU oracle, c3-c5
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/s4h
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/s4h/bench_c2.json 2> gpurun_out/s4h/bench_c2.err; echo c2 rc=$?
python -c "import json; d=json.load(open('gpurun_out/s4h/bench_c2.json')); print('c2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, round(d['roofline']['frac'],3))"
for c in c3 c4 c5; do
  timeout 1500 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/s4h/bench_$c.json 2> gpurun_out/s4h/bench_$c.err; echo $c rc=$?
  python -c "import json; d=json.load(open('gpurun_out/s4h/bench_$c.json')); print('$c', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, round(d['roofline']['frac'],3))"
done
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
