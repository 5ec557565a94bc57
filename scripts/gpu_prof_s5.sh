# session-5: c2 launch list (planner + coarse changes), planner blocks-per-SM check, reference arm
mkdir -p gpurun_out/s5
export PATH=/usr/local/cuda/bin:$PATH
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s5/launches_c2.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches rc=$?
python scripts/launch_summary.py gpurun_out/s5/launches_c2.csv > gpurun_out/s5/launches_c2_summary.txt; tail -15 gpurun_out/s5/launches_c2_summary.txt
for c in c2 c3; do
  MV_PLAN_BPS=1 timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/s5/bps1_$c.json 2>/dev/null
  python -c "import json; d=json.load(open('gpurun_out/s5/bps1_$c.json')); print('bps1 $c', round(d['value']), {a: round(b,3) for a,b in d['stage_ms'].items()})"
done
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/s5/bench_ref.json 2> gpurun_out/s5/bench_ref.err; echo ref rc=$?
