O=gpurun_out/q_o; mkdir -p $O
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo pytest=$?; tail -3 $O/pytest.log
for c in c3 c2 c5 c4; do timeout 600 python bench.py --config $c --no-cpu-baseline > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
