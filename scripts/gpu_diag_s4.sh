# session-4 diagnosis: which scan role bounds phase B?  MV_SCAN_DEBUG bits: 1 no emission stores,
# 2 no epilogue math, 4 no query-plane gather (results invalid; timings only)
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/d4
timeout 900 python -m pytest tests -m gpu -x -q --timeout 600 -k "large_k or c1 or sq8 or merge" 2>&1 | tail -3
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/d4/b_$2_$3.json 2> gpurun_out/d4/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/d4/b_$2_$3.json')); print('$1 $2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()})" || tail -3 gpurun_out/d4/b_$2_$3.err
}
for c in c2 c3; do
  run MV_SCAN_DEBUG=0 $c d0
  run MV_SCAN_DEBUG=1 $c d1
  run MV_SCAN_DEBUG=3 $c d3
  run MV_SCAN_DEBUG=7 $c d7
  run MV_SCAN_DEBUG=4 $c d4
done
run MV_SCAN_DEBUG=0 c4 sel
run MV_SQ8_QC=32 c3 qc32
run MV_SQ8_QC=16 c3 qc16
run MV_FLAT_QC=64 c2 qc64
run MV_FLAT_QC=48 c2 qc48
MV_SCAN_TRACE=1 timeout 300 python bench.py --config c2 --steps 1 --warmup 0 --no-cpu-baseline 2> gpurun_out/d4/trace_c2.txt > /dev/null
MV_SCAN_TRACE=1 timeout 300 python bench.py --config c3 --steps 1 --warmup 0 --no-cpu-baseline 2> gpurun_out/d4/trace_c3.txt > /dev/null
export PATH=/usr/local/cuda/bin:$PATH
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"k_scan_tc|k_final|k_tau" -s 12 -c 4 -o gpurun_out/d4/full_c3 python bench.py --config c3 --steps 1 --warmup 2 --no-cpu-baseline > gpurun_out/d4/ncu_c3.log 2>&1; echo full rc=$?
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"k_final_big|k_scan_tc" -s 8 -c 4 -o gpurun_out/d4/full_c4 python bench.py --config c4 --steps 1 --warmup 2 --no-cpu-baseline > gpurun_out/d4/ncu_c4.log 2>&1; echo full4 rc=$?
timeout 1200 ncu --set full --import-source on --clock-control none -k regex:"k_coarse_gemm|k_scan_tc|k_final_warp|k_probe_select|k_plan" -s 34 -c 7 -o gpurun_out/d4/full_c2 python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/d4/ncu_c2.log 2>&1; echo full2 rc=$?
