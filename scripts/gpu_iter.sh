O=gpurun_out/q_an; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "c1 or flat_l2 or sq8 or large_k" > $O/pytest.log 2>&1; echo pytest=$?; tail -1 $O/pytest.log
for c in c2 c4 c5 c3; do timeout 900 python scripts/sweep_opts.py --config $c --sets "" > $O/sweep_$c.txt 2>&1; grep -v "^\[bench" $O/sweep_$c.txt; done
