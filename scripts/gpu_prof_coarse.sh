python -c "import __graft_entry__ as g; g.build()" || exit 1
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_coarse_gemm|k_scan_tc" -s 9 -c 3 -o gpurun_out/full_c2b python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1; echo full rc=$?
