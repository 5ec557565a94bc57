O=gpurun_out/q_e; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_filtering.py -x -q -p no:cacheprovider > $O/pytest_f4.log 2>&1; echo f4=$?; tail -3 $O/pytest_f4.log
timeout 900 python scripts/sweep_opts.py --config c4 --sets "" "flat_qc=80" "flat_qc=64" "flat_qc=48" > $O/sweep_c4.txt 2>&1; echo s4=$?
timeout 900 python scripts/sweep_opts.py --config c2 --sets "" "flat_qc=80" "flat_qc=64" "flat_qc=48" > $O/sweep_c2.txt 2>&1; echo s2=$?
timeout 900 ncu --profile-from-start off --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv python scripts/prof_search.py --config c4 > $O/launches_c4.csv 2>/dev/null; python scripts/ncu_summary.py $O/launches_c4.csv > $O/launches_c4_summary.txt
