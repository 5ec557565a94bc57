# session-5: parity + bench after the slimmer coarse epilogue
mkdir -p gpurun_out/w11
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/w11/pytest.log 2>&1; tail -1 gpurun_out/w11/pytest.log
for c in c2 c3 c4 c5; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/w11/b_$c.json 2> gpurun_out/w11/b_$c.err
  python -c "import json; d=json.load(open('gpurun_out/w11/b_$c.json')); print('$c', round(d['value']), {a: round(b,3) for a,b in d['stage_ms'].items()})" || tail -3 gpurun_out/w11/b_$c.err
done
