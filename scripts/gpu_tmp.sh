O=gpurun_out/q_k; mkdir -p $O
L=paper_conf_sigmod_wangygjxlwglxyy21_b200/libmv.so
timeout 900 python -m pytest tests -m "gpu and not slow" -x -q -p no:cacheprovider > $O/pytest.log 2>&1; echo pytest=$?; tail -3 $O/pytest.log
timeout 900 python scripts/sweep_opts.py --config c4 --sets "" "large_k_select=2" "large_k_select=3" > $O/sweep_c4.txt 2>&1; echo s4=$?
for v in nommaepi nogather nothing; do
  cp exp/lib_$v.so $L
  for c in c5 c3 c4; do timeout 600 python scripts/sweep_opts.py --config $c --steps 5 --sets "" 2>&1 | grep -v "^\[bench" | sed "s/^/$v /" >> $O/exp.txt; done
done
cp exp/lib_prod.so $L
