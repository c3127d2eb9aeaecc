set -x
mkdir -p gpurun_out/r01b
M=gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_elapsed.avg.per_second,gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r01b/launches.csv python bench.py --steps 1 --warmup 3 --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample > gpurun_out/r01b/launches_bench.log 2>&1
timeout 600 ncu --metrics $M --clock-control none -k regex:update_kernel --csv --log-file gpurun_out/r01b/c2_update.csv python studies/probes/c2_one.py 8192 16384 > gpurun_out/r01b/c2.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_kernel --launch-skip 30 --launch-count 1 -o gpurun_out/r01b/update_full python bench.py --steps 1 --warmup 2 --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample > gpurun_out/r01b/full_bench.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:"split_cols_t|colmax_tile_k|split_rows_f16" --launch-skip 3 --launch-count 3 -o gpurun_out/r01b/stage_full python bench.py --steps 1 --warmup 1 --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample > gpurun_out/r01b/stage_bench.log 2>&1
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:update_kernel --csv --log-file gpurun_out/r01b/update_traffic.csv python bench.py --steps 1 --warmup 0 --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample > gpurun_out/r01b/traffic_bench.log 2>&1
ls -la gpurun_out/r01b
