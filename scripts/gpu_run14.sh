timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | tail -1
for d in 0 32; do MV_SCAN_DEBUG=$d timeout 300 python bench.py --steps 50 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('dbg=$d', round(d['value']), 'qps', {a: round(b,3) for a,b in d['stage_ms'].items()})"; done
