O=gpurun_out/q_ab; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "flat or c1 or options or large_k or edge" > $O/pytest.log 2>&1; echo pytest=$?; tail -2 $O/pytest.log
for c in c4 c2; do timeout 900 python scripts/sweep_opts.py --config $c --sets "" > $O/sweep_$c.txt 2>&1; grep -v "^\[bench" $O/sweep_$c.txt; done
