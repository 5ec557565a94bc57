for d in 0 1 3 7 15; do MV_SCAN_DEBUG=$d timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('dbg=$d scan', round(d['stage_ms']['scan'],3))"; done
MV_SCAN_TRACE=1 timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "\[trace\]" | grep epi | head -4 | cut -c1-400
