# profiles for this round: launch list (per-kernel device times) + full capture of scan and coarse
export PATH=/usr/local/cuda/bin:$PATH
mkdir -p gpurun_out/prof
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/prof/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches rc=$?
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_scan_tc|k_coarse_tc|k_final_select" -s 6 -c 3 -o gpurun_out/prof/full python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo full rc=$?
timeout 900 python bench.py > gpurun_out/prof/bench_c2.json 2> gpurun_out/prof/bench_c2.err; echo bench rc=$?
