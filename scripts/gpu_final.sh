#!/bin/bash
# The round's measurement set on one B200: ncu launch lists (-> profiles/scan_traffic.json and
# coarse_tensor_pipe.json, read by bench.py), the full GPU test suite, smoke, the bench lines of
# every config, the reference arm, the rounds ablation, ncu full captures of the scan.
T=${1:-final}
O=gpurun_out/$T
mkdir -p $O
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed
for c in c4 c3 c5 c2; do
  timeout 900 ncu --profile-from-start off --metrics $M --clock-control none --csv python scripts/prof_search.py --config $c > $O/launches_$c.csv 2> $O/launches_$c.err; echo launches_$c=$?
  python scripts/ncu_summary.py $O/launches_$c.csv > $O/launches_${c}_summary.txt 2>&1
done
python scripts/make_profile_tables.py $T c4=$O/launches_c4.csv c3=$O/launches_c3.csv c5=$O/launches_c5.csv c2=$O/launches_c2.csv > $O/tables.txt 2>&1; echo tables=$?
cp profiles/scan_traffic.json profiles/coarse_tensor_pipe.json $O/
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo smoke=$?
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_gpu.log 2>&1; echo pytest=$?; tail -3 $O/pytest_gpu.log
timeout 900 python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo bench=$?
for c in c2 c3 c5 c3pq; do timeout 900 python bench.py --config $c --no-cpu-baseline > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
timeout 900 python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.err; echo ref=$?
timeout 900 python scripts/rounds_ablation.py > $O/rounds.json 2> $O/rounds.err; echo rounds=$?
for c in c4 c3; do
  timeout 900 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:k_scan_tc --launch-skip 1 --launch-count 1 -o $O/full_scanB_$c python scripts/prof_search.py --config $c > $O/full_scanB_$c.log 2>&1; echo full_$c=$?
  ncu -i $O/full_scanB_$c.ncu-rep --page raw --csv > $O/full_scanB_${c}_raw.csv 2>/dev/null
done
