export PATH=/usr/local/cuda/bin:$PATH
timeout 300 compute-sanitizer --tool memcheck python scripts/dbg_small.py 10 2>&1 | grep -v "^=========     Host Frame" | head -40
timeout 300 compute-sanitizer --tool memcheck python scripts/dbg_small.py 100 2>&1 | grep -v "Host Frame" | head -20
