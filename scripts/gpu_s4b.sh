# session-4: barrier-free count publish + the seeding sample-size rule; full GPU tests and c2-c5 lines
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/s4b
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 2>&1 | tail -2
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/s4b/b_$2_$3.json 2> gpurun_out/s4b/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/s4b/b_$2_$3.json')); print('$1 $2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, round(d['roofline']['frac'],3))" || tail -3 gpurun_out/s4b/b_$2_$3.err
}
run MV_NEED=0 c2 x
run MV_NEED=0 c3 x
run MV_NEED=0 c4 x
run MV_NEED=0 c5 x
MV_SCAN_TRACE=1 timeout 300 python bench.py --config c2 --steps 1 --warmup 0 --no-cpu-baseline 2> gpurun_out/s4b/trace_c2.txt > /dev/null
