O=gpurun_out/q_ag; mkdir -p $O
timeout 900 python scripts/sweep_opts.py --config c5 --sets "" "need=1000" "need=1000,capa=512" "capa=512" > $O/sweep_c5.txt 2>&1; grep -v "^\[bench" $O/sweep_c5.txt
timeout 900 python scripts/sweep_opts.py --config c3 --sets "" "need=600" "need=1200" "capa=128" > $O/sweep_c3.txt 2>&1; grep -v "^\[bench" $O/sweep_c3.txt
timeout 900 python scripts/sweep_opts.py --config c2 --sets "" "need=100" "capa=256" > $O/sweep_c2.txt 2>&1; grep -v "^\[bench" $O/sweep_c2.txt
