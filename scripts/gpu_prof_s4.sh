# session-4 profiles: default bench line (c2, with the CPU oracle baseline), c3/c4/c5 lines, the ncu
# launch list of a c2 run and one ncu --set full capture of a c2 search's main kernels
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/s4
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 2>&1 | tail -2
timeout 900 python bench.py > gpurun_out/s4/bench_c2.json 2> gpurun_out/s4/bench_c2.err; echo c2 rc=$?
for c in c3 c4 c5; do
  timeout 1500 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/s4/bench_$c.json 2> gpurun_out/s4/bench_$c.err; echo $c rc=$?
done
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/s4/launches_c2.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline > /dev/null 2>&1; echo launches rc=$?
python scripts/launch_summary.py gpurun_out/s4/launches_c2.csv > gpurun_out/s4/launches_c2_summary.txt
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"k_coarse_gemm|k_scan_tc|k_final_warp|k_probe_select|k_plan" -s 24 -c 6 -o gpurun_out/s4/full_c2 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/s4/ncu_full.log 2>&1; echo full rc=$?
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/s4/bench_ref.json 2> gpurun_out/s4/bench_ref.err; echo ref rc=$?
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2
