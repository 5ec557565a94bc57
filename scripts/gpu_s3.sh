python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | tail -2
for c in c2 c3; do
  for seed in 1 0; do
  for d in 0 1 3 7; do
    MV_SEED=$seed MV_SCAN_DEBUG=$d timeout 300 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('$c seed=$seed dbg=$d', round(d['value']), d['config']['recall@10'], {a: round(b,3) for a,b in d['stage_ms'].items()})"
  done
  MV_SEED=$seed MV_SCAN_TRACE=1 MV_SCAN_DEBUG=64 timeout 300 python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline 2>&1 >/dev/null | grep events | tail -1
  done
done
timeout 600 python bench.py --config c4 --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
python -c "import json; d=json.load(open('gpurun_out/bench_c4.json')); print('c4', round(d['value']), 'qps', d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, 'frac', round(d['roofline']['frac'],3), d['index']['last_scan'], d['index']['last_coarse'])" || tail -5 gpurun_out/bench_c4.err
