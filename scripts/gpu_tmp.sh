O=gpurun_out/q_w; mkdir -p $O
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo pytest=$?; tail -2 $O/pytest.log
for c in c5 c4 c3 c2; do timeout 900 python scripts/sweep_opts.py --config $c --sets "" > $O/sweep_$c.txt 2>&1; grep -v "^\[bench" $O/sweep_$c.txt; done
