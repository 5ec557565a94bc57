python -c "import __graft_entry__ as g; g.build()" || exit 1
MV_SCAN_TRACE=1 timeout 600 python bench.py --config c2 --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/trace2.json 2> gpurun_out/trace2.err
