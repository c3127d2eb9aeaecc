set -x
O=gpurun_out/r02h; mkdir -p $O
B="python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0"
for cfg in "0 0" "1 0" "0 1" "1 1" "0 2"; do
  set -- $cfg
  timeout 300 $B --raster-snake $1 --l2-hint-b $2 > $O/bench_s$1_h$2.json 2>&1
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:update_acc -s 6 -c 2 --csv python bench.py --steps 1 --warmup 1 --no-hetero --no-cpu-baseline --e2e-steps 0 --no-sample --raster-snake $1 --l2-hint-b $2 > $O/ncu_s$1_h$2.csv 2>&1
done
for G in 12 20; do
  timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:update_acc -s 6 -c 2 --csv python bench.py --steps 1 --warmup 1 --no-hetero --no-cpu-baseline --e2e-steps 0 --no-sample --raster-group $G --raster-snake 1 > $O/ncu_g$G.csv 2>&1
  timeout 300 $B --raster-group $G --raster-snake 1 > $O/bench_g$G.json 2>&1
done
