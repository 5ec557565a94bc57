for c in 0 1 3; do for d in 0 1 3 7; do
  MV_COARSE_DEBUG=$c MV_SCAN_DEBUG=$d timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>/dev/null > /tmp/o.json; python -c "import json,sys; d=json.load(open('/tmp/o.json')); s=d['stage_ms']; print('coarse_dbg=$c scan_dbg=$d', 'coarse', round(s['coarse'],3), 'scan', round(s['scan'],3))" 2>/dev/null || echo "fail $c $d"
done; done
