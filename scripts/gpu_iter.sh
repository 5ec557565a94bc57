O=gpurun_out/q_af; mkdir -p $O
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo pytest=$?; tail -2 $O/pytest.log
for i in 1 2; do timeout 900 python scripts/sweep_opts.py --config c4 --sets "" "large_k_select=4" > $O/sweep_c4_$i.txt 2>&1; grep -v "^\[bench" $O/sweep_c4_$i.txt; done
