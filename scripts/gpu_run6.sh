export PATH=/usr/local/cuda/bin:$PATH
timeout 300 compute-sanitizer --tool memcheck python scripts/dbg_small.py 10 2>&1 | grep -v "Host Frame" | tail -3
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q --timeout 300 2>&1 | grep -E "passed|failed|Error|error|assert" | head -20
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print(round(d['value']), 'qps', d['ms_per_step'], d['stage_ms'], d['index']['last_scan'], d['index']['last_coarse'], d['config']['recall@10'])"
