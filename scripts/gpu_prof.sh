# ncu capture of the scan kernel on the c2 bench (1 step, no cpu baseline); launch list too
export PATH=/usr/local/cuda/bin:$PATH
timeout 300 python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_p.json 2>gpurun_out/bench_p.err; cat gpurun_out/bench_p.json | python -c "import json,sys; d=json.load(sys.stdin); print(d['index'], d['stage_ms'], d['ms_per_step'])"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches rc=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:k_scan_tc -s 3 -c 1 -o gpurun_out/scan_tc python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_scan.log 2>&1; echo ncu rc=$?
tail -3 gpurun_out/ncu_scan.log
