O=gpurun_out/r02z; mkdir -p $O
B="python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0"
for i in 1 2; do
  timeout 300 $B > $O/f2_$i.json 2>&1
  timeout 300 $B --fuse 4 > $O/f4_$i.json 2>&1
  timeout 300 $B --fuse 3 > $O/f3_$i.json 2>&1
done
timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:update_acc -s 4 -c 2 --csv --log-file $O/ncu_f4.csv python bench.py --steps 1 --warmup 1 --no-hetero --no-cpu-baseline --e2e-steps 0 --no-sample --fuse 4 > /dev/null 2>&1
timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:update_acc -s 6 -c 2 --csv --log-file $O/ncu_f2.csv python bench.py --steps 1 --warmup 1 --no-hetero --no-cpu-baseline --e2e-steps 0 --no-sample > /dev/null 2>&1
