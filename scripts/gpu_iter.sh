O=gpurun_out/q_ah; mkdir -p $O
timeout 900 python scripts/sweep_opts.py --config c4 --sets "" "need=11000" "need=13000" "need=20000" "capa=768" "capa=1536" > $O/sweep_c4.txt 2>&1; grep -v "^\[bench" $O/sweep_c4.txt
timeout 900 python scripts/sweep_opts.py --config c3pq --sets "" > $O/sweep_c3pq.txt 2>&1; grep -v "^\[bench" $O/sweep_c3pq.txt
