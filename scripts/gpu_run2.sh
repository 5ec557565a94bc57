nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 120 ./tests/cuda/umma_selftest | tail -1
timeout 240 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -3; echo smoke rc=${PIPESTATUS[0]}
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | tail -25
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench2.json 2> gpurun_out/bench2.err; echo bench rc=$?
tail -3 gpurun_out/bench2.err; cat gpurun_out/bench2.json
