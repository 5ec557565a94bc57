python -c "import __graft_entry__ as g; g.build()" || exit 1
export PATH=/usr/local/cuda/bin:$PATH
timeout 1500 ncu --set full --import-source on --clock-control none -k regex:"k_scan_tc" -s 3 -c 1 -o gpurun_out/full_c5 python bench.py --config c5 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_c5.log 2>&1; echo full rc=$?
