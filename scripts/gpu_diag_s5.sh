# session-5 coarse diagnosis: epilogue off (2) / score stores off (4), timing only
mkdir -p gpurun_out/w9
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/w9/b_$2_$3.json 2> gpurun_out/w9/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/w9/b_$2_$3.json')); print('$1 $2', round(d['value']), {a: round(b,3) for a,b in d['stage_ms'].items()})" || tail -3 gpurun_out/w9/b_$2_$3.err
}
for c in c3 c5; do
run "MV_COARSE_DEBUG=4" $c nost
run "MV_COARSE_DEBUG=2" $c noepi
done
