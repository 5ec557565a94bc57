# session-4 final-state profiles: GPU tests, bench lines c2 (with the CPU oracle) .. c5, the c2 ncu
# launch list, ncu --set full of one c2 search and of c4's large-k selects
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/s4d
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/s4d/bench_c2.json 2> gpurun_out/s4d/bench_c2.err; echo c2 rc=$?
python -c "import json; d=json.load(open('gpurun_out/s4d/bench_c2.json')); print('c2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, round(d['roofline']['frac'],3))"
for c in c3 c4 c5; do
  timeout 1500 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/s4d/bench_$c.json 2> gpurun_out/s4d/bench_$c.err; echo $c rc=$?
  python -c "import json; d=json.load(open('gpurun_out/s4d/bench_$c.json')); print('$c', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, round(d['roofline']['frac'],3))"
done
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s4d/launches_c2.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches rc=$?
python scripts/launch_summary.py gpurun_out/s4d/launches_c2.csv > gpurun_out/s4d/launches_c2_summary.txt
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"k_coarse_gemm|k_scan_tc|k_final_warp|k_probe_select|k_plan" -s 34 -c 7 -o gpurun_out/s4d/full_c2 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/s4d/ncu_c2.log 2>&1; echo full2 rc=$?
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"k_final_big|k_scan_tc" -s 8 -c 4 -o gpurun_out/s4d/full_c4 python bench.py --config c4 --steps 1 --warmup 2 --no-cpu-baseline > gpurun_out/s4d/ncu_c4.log 2>&1; echo full4 rc=$?
