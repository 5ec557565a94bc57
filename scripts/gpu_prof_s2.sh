# ncu: full capture of one search's main kernels (c2), plus the launch list of one bench step
python -c "import __graft_entry__ as g; g.build()" || exit 1
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_coarse_tc|k_scan_tc|k_final_warp" -s 15 -c 5 -o gpurun_out/full_c2 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1; echo full rc=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_c2.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches rc=$?
