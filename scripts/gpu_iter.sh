O=gpurun_out/q_ak; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_pq.py -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo pytest=$?; tail -2 $O/pytest.log
timeout 900 python scripts/sweep_opts.py --config c3pq --sets "" > $O/sweep_c3pq.txt 2>&1; grep -v "^\[bench" $O/sweep_c3pq.txt
