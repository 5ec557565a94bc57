MV_SCAN_TRACE=1 timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "\[trace\]" | head -8
MV_SCAN_TRACE=1 MV_SCAN_DEBUG=15 timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "\[trace\]" | head -8
