for d in 7 15; do MV_SCAN_DEBUG=$d timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null > /tmp/o.json; python -c "import json; d=json.load(open('/tmp/o.json')); print('dbg=$d scan', round(d['stage_ms']['scan'],3))"; done
MV_SCAN_PROF=1 MV_SCAN_DEBUG=15 timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "scan prof" | tail -13
