#!/bin/bash
# The round's measurement set (one gpurun call): full-size parity, the default bench line and the
# other configs, the reference arm, and the ncu evidence (launch lists + scan DRAM traffic).
set -x
O=gpurun_out/r02
mkdir -p $O
timeout 1500 python -m pytest tests -m "gpu and slow" -q -p no:cacheprovider > $O/pytest_slow.log 2>&1; echo slow_rc=$?
python bench.py > $O/bench_default.json 2> $O/bench_default.err; echo bench_rc=$?
for c in c2 c3 c5; do python bench.py --config $c --no-cpu-baseline > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
python bench.py --impl reference > $O/bench_reference.json 2> $O/bench_reference.err; echo ref=$?
for c in c4 c2 c3; do
  ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none --csv python scripts/prof_search.py --config $c > $O/ncu_launches_$c.csv 2> $O/ncu_launches_$c.err; echo ncu_$c=$?
done
