# session-4: 1024-thread large-k select; seeding-extremes parity tests; c4 lines
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/s4f
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -k "large_k or merge or edge or seeding or c1" 2>&1 | tail -3
for c in c4; do
  timeout 1500 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/s4f/bench_$c.json 2> gpurun_out/s4f/bench_$c.err; echo $c rc=$?
  python -c "import json; d=json.load(open('gpurun_out/s4f/bench_$c.json')); print('$c', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, round(d['roofline']['frac'],3))"
done
