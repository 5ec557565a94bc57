#!/bin/bash
# Iteration run: GPU parity tests (not slow), then bench lines for the given configs.
# Usage: bash scripts/gpu_quick.sh TAG "c4 c2 c3" [extra sweep args...]
T=$1; CFGS=$2; shift 2
O=gpurun_out/q_$T
mkdir -p $O
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo pytest=$?; tail -2 $O/pytest.log
for c in $CFGS; do timeout 600 python bench.py --config $c --no-cpu-baseline > $O/bench_$c.json 2> $O/bench_$c.err; echo $c=$?; done
if [ $# -gt 0 ]; then timeout 900 python scripts/sweep_opts.py "$@" > $O/sweep.txt 2>&1; echo sweep=$?; fi
