#!/bin/bash
# ncu evidence for one round session: per-search launch lists (time, DRAM bytes, tensor pipe) of
# c4/c3/c5/c2, and --set full captures of the phase-B scan (c3, c5, c4) and the coarse GEMM (c3).
# Usage: bash scripts/gpu_ncu.sh TAG
T=${1:-s}
O=gpurun_out/ncu_$T
mkdir -p $O
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed
for c in c4 c3 c5 c2; do
  timeout 900 ncu --profile-from-start off --metrics $M --clock-control none --csv python scripts/prof_search.py --config $c > $O/launches_$c.csv 2> $O/launches_$c.err; echo launches_$c=$?
  python scripts/ncu_summary.py $O/launches_$c.csv > $O/launches_${c}_summary.txt 2>&1
done
for c in c3 c5 c4; do
  timeout 900 ncu --profile-from-start off --set full --import-source on --clock-control none -k regex:k_scan_tc --launch-skip 1 --launch-count 1 -o $O/full_scanB_$c python scripts/prof_search.py --config $c > $O/full_scanB_$c.log 2>&1; echo full_$c=$?
  ncu -i $O/full_scanB_$c.ncu-rep --page raw --csv > $O/full_scanB_${c}_raw.csv 2>/dev/null
done
timeout 900 ncu --profile-from-start off --set full --clock-control none -k regex:k_coarse_qm --launch-count 2 -o $O/full_coarse_c3 python scripts/prof_search.py --config c3 > $O/full_coarse_c3.log 2>&1; echo coarse=$?
ncu -i $O/full_coarse_c3.ncu-rep --page raw --csv > $O/full_coarse_c3_raw.csv 2>/dev/null
