timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | grep -E "passed|failed" | head -3
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(round(d['value']), 'qps', d['ms_per_step'], d['stage_ms'])"
MV_SCAN_TRACE=1 timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "\[trace\]" | grep epi | head -4
