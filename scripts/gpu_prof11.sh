export PATH=/usr/local/cuda/bin:$PATH
MV_SCAN_DEBUG=15 timeout 600 ncu --set full --import-source on --clock-control none -k regex:k_scan_tc -s 2 -c 1 -o gpurun_out/skel15 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo rc=$?
