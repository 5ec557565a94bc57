timeout 300 python scripts/dbg_sq8.py 2>&1 | grep maxabs
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | grep -E "passed|failed|Error|error|assert" | head -20
for d in 0 1; do
  MV_SCAN_DEBUG=$d timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('dbg=$d', round(d['stage_ms']['scan'],3), 'ms scan', round(d['value']), 'qps', d['index']['last_scan'], d['config']['recall@10'])"
done
