# session-4 sweep 4: coarse GEMM query-block size x centroid split on the large-nlist configs
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/w7
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/w7/b_$2_$3.json 2> gpurun_out/w7/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/w7/b_$2_$3.json')); print('$1 $2', round(d['value']), {a: round(b,3) for a,b in d['stage_ms'].items()})" || tail -3 gpurun_out/w7/b_$2_$3.err
}
run "MV_X=0" c5 base
run "MV_COARSE_NQB=128 MV_COARSE_CS=4" c5 a
run "MV_COARSE_NQB=128 MV_COARSE_CS=16" c5 b
run "MV_COARSE_NQB=64 MV_COARSE_CS=8" c5 c
run "MV_COARSE_NQB=128 MV_COARSE_CS=32" c5 d
run "MV_X=0" c3 base
run "MV_COARSE_NQB=128 MV_COARSE_CS=4" c3 a
run "MV_COARSE_NQB=128 MV_COARSE_CS=16" c3 b
run "MV_COARSE_NQB=64 MV_COARSE_CS=8" c3 c
