python -c "import __graft_entry__ as g; g.build()" || exit 1
MV_SCAN_TRACE=1 timeout 1500 python bench.py --config c5 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/trace5.json 2> gpurun_out/trace5.err
grep -c trace gpurun_out/trace5.err
