timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | tail -5
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench3.json 2>gpurun_out/bench3.err; python -c "import json; d=json.load(open('gpurun_out/bench3.json')); print(d['value'], d['index']['last_scan'], d['stage_ms'], d['roofline']['frac'])"
timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_scan_tc -s 3 -c 1 -o gpurun_out/scan_tc2 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_scan2.log 2>&1; echo ncu rc=$?
