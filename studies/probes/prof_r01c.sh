# Profiles of the F16I8 default (round 1, third pass): launch list, one --set full
# capture of the update, DRAM traffic of every update launch of one step.
set -x
D=gpurun_out/r01c; mkdir -p $D
B="python bench.py --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $D/launches.csv $B --steps 1 --warmup 3 > $D/launches_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_hyb_kernel --launch-skip 30 --launch-count 1 -o $D/update_full $B --steps 1 --warmup 2 > $D/full_bench.log 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,sm__cycles_elapsed.avg.per_second --clock-control none -k regex:update_hyb_kernel --csv --log-file $D/update_traffic.csv $B --steps 1 --warmup 0 > $D/traffic_bench.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:"split_cols_t|colmax_tile_k|split_rows_f16" --launch-skip 3 --launch-count 3 -o $D/stage_full $B --steps 1 --warmup 1 > $D/stage_bench.log 2>&1
ls -la $D
