for d in 15 0; do MV_SCAN_TRACE=1 MV_SCAN_DEBUG=$d timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "\[cta\]" | head -1 > gpurun_out/cta_$d.txt; done
