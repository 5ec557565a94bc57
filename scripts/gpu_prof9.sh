export PATH=/usr/local/cuda/bin:$PATH
M="dram__bytes_read.sum,dram__bytes_write.sum,lts__t_bytes.sum,gpu__time_duration.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,lts__throughput.avg.pct_of_peak_sustained_elapsed,dram__throughput.avg.pct_of_peak_sustained_elapsed,sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_elapsed,smsp__warps_active.avg.per_cycle_active"
for d in 7 0; do
MV_SCAN_DEBUG=$d timeout 600 ncu --metrics $M --clock-control none -k regex:"k_scan_tc|k_coarse_tc|k_final|k_bucket|k_scan_single|k_count|k_work|k_query_tot|k_pair_off|k_qplanes|k_hilo|k_row_prep" -s 14 -c 14 --csv python bench.py --steps 1 --warmup 3 --no-cpu-baseline 2>/dev/null > gpurun_out/scan_d$d.csv; echo rc=$?
done
