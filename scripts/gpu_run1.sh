# every step bounded by its own timeout (a hung kernel must not eat the gpurun budget)
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
timeout 240 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -5; echo smoke rc=${PIPESTATUS[0]}
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | tail -25
timeout 600 python bench.py --steps 5 --warmup 3 > gpurun_out/bench1.json 2> gpurun_out/bench1.err; echo bench rc=$?
tail -5 gpurun_out/bench1.err; cat gpurun_out/bench1.json
