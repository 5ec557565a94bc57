export PATH=/usr/local/cuda/bin:$PATH
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | grep -E "passed|failed|Error|error|assert" | head -20
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 600 ncu --set full --import-source on --clock-control none -k regex:"k_coarse_tc|k_scan_tc" -s 2 -c 2 -o gpurun_out/prof7 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu7.log 2>&1; echo ncu rc=$?
