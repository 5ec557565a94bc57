# session-4 sweep 3: rows per list of the seeding sample (MV_CAPA) at the rule's sample size
python -c "import __graft_entry__ as g; g.build()" || exit 1
mkdir -p gpurun_out/w6
run() {
  env $1 timeout 900 python bench.py --config $2 --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/w6/b_$2_$3.json 2> gpurun_out/w6/b_$2_$3.err
  python -c "import json; d=json.load(open('gpurun_out/w6/b_$2_$3.json')); print('$1 $2', round(d['value']), d['config'].get('recall@10'), {a: round(b,3) for a,b in d['stage_ms'].items()})" || tail -3 gpurun_out/w6/b_$2_$3.err
}
run MV_CAPA=128 c4 c128
run MV_CAPA=256 c4 c256
run MV_CAPA=512 c4 c512
run MV_CAPA=128 c3 c128
run MV_CAPA=256 c3 c256
run MV_CAPA=64 c5 c64
run MV_CAPA=256 c5 c256
