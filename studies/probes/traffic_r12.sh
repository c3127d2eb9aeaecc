D=gpurun_out/r01d; mkdir -p $D
timeout 300 python -m pytest tests/test_gpu_f16i8.py tests/test_gpu_pmm.py -x -q 2>&1 | tail -2
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:update_hyb_kernel --csv --log-file $D/update_traffic.csv python bench.py --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample --steps 1 --warmup 0 > $D/traffic_bench.log 2>&1
timeout 900 python bench.py > $D/bench.json 2> $D/bench.err
tail -c 400 $D/bench.json
