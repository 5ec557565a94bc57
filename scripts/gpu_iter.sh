O=gpurun_out/q_al; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "large_k or options" > $O/pytest.log 2>&1; echo pytest=$?; tail -2 $O/pytest.log
timeout 900 python scripts/sweep_opts.py --config c4 --sets "" > $O/sweep_c4.txt 2>&1; grep -v "^\[bench" $O/sweep_c4.txt
