python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/s3
export PATH=/usr/local/cuda/bin:$PATH
# skip the add path's 16 row blocks (coarse GEMM + select each) and 3 warm-up searches (7 matches each)
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"k_coarse_gemm|k_scan_tc|k_final_warp|k_probe_select|k_plan" -s 53 -c 7 -o gpurun_out/s3/full_c2b python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/s3/ncu_full_b.log 2>&1; echo full rc=$?
