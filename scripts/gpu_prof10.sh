for d in 0 7; do echo "== dbg $d"; MV_SCAN_PROF=1 MV_SCAN_DEBUG=$d timeout 300 python bench.py --steps 1 --warmup 0 --no-cpu-baseline 2>&1 | grep "scan prof" | tail -13; done
