O=gpurun_out/q_am; mkdir -p $O
timeout 900 python scripts/sweep_opts.py --config c4 --sets "" "flat_qc=112" "flat_qc=128" "flat_qc=80" > $O/sweep_c4.txt 2>&1; grep -v "^\[bench" $O/sweep_c4.txt
timeout 900 python scripts/sweep_opts.py --config c5 --sets "" "sq8_qc=48" "sq8_qc=32" > $O/sweep_c5.txt 2>&1; grep -v "^\[bench" $O/sweep_c5.txt
timeout 900 python scripts/sweep_opts.py --config c2 --sets "" "flat_qc=112" "flat_qc=64" > $O/sweep_c2.txt 2>&1; grep -v "^\[bench" $O/sweep_c2.txt
