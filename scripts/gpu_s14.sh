python -c "import __graft_entry__ as g; g.build()" || exit 1
run() {
  env $1 timeout 600 python bench.py --config ${2:-c2} --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/x.json 2> gpurun_out/x.err
  python -c "import json; d=json.load(open('gpurun_out/x.json')); print('$1 ${2:-c2}', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()}, d['index']['last_scan'])" || tail -3 gpurun_out/x.err
}
run MV_SCAN_DEBUG=6
run MV_SCAN_DEBUG=22
run MV_SCAN_DEBUG=38
run MV_SCAN_DEBUG=54
run MV_SCAN_DEBUG=62
export PATH=/usr/local/cuda/bin:$PATH
timeout 900 ncu --set full --import-source on --clock-control none -k regex:"k_scan_qm" -s 6 -c 2 -o gpurun_out/full_qm python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/ncu_full.log 2>&1; echo full rc=$?
