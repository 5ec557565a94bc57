# session-5 sweep: coarse GEMM epilogue warps x TMEM accumulators (parity first at the extreme setting)
mkdir -p gpurun_out/w8
MV_COARSE_EPI=16 MV_COARSE_NACC=4 timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/w8/pytest_e16a4.log 2>&1; tail -1 gpurun_out/w8/pytest_e16a4.log
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/w8/b_$2_$3.json 2> gpurun_out/w8/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/w8/b_$2_$3.json')); print('$1 $2', round(d['value']), {a: round(b,3) for a,b in d['stage_ms'].items()})" || tail -3 gpurun_out/w8/b_$2_$3.err
}
for c in c2 c5 c3; do
run "MV_X=0" $c base
run "MV_COARSE_NACC=4" $c a4
run "MV_COARSE_EPI=12" $c e12
run "MV_COARSE_EPI=16" $c e16
run "MV_COARSE_EPI=12 MV_COARSE_NACC=4" $c e12a4
run "MV_COARSE_EPI=16 MV_COARSE_NACC=4" $c e16a4
done
