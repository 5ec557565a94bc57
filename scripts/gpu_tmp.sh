O=gpurun_out/q_m; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_pq.py -x -q -p no:cacheprovider > $O/pytest_pq.log 2>&1; echo pq=$?; tail -15 $O/pytest_pq.log
timeout 900 python -m pytest tests -m "gpu and not slow" -q -p no:cacheprovider > $O/pytest.log 2>&1; echo pytest=$?; tail -3 $O/pytest.log
timeout 600 python bench.py --config c4 --no-cpu-baseline > $O/bench_c4.json 2> $O/bench_c4.err; echo c4=$?
