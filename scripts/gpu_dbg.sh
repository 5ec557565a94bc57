for d in 0 1 3 7 4; do
  MV_SCAN_DEBUG=$d timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null | python -c "import json,sys; d=json.load(sys.stdin); print('dbg=$d', round(d['stage_ms']['scan'],3), 'ms scan')"
done
