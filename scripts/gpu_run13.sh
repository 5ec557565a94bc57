timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | grep -E "passed|failed|Error" | head -5
timeout 900 python bench.py > gpurun_out/bench13.json 2> gpurun_out/bench13.err; echo bench rc=$?; tail -2 gpurun_out/bench13.err
