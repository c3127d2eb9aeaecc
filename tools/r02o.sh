O=gpurun_out/r02o; mkdir -p $O
B="python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0"
for i in 1 2; do
  timeout 300 $B > $O/f2_g16_$i.json 2>&1
  timeout 300 $B --fuse 4 --raster-group 8 > $O/f4_g8_$i.json 2>&1
  timeout 300 $B --fuse 4 --raster-group 6 > $O/f4_g6_$i.json 2>&1
  timeout 300 $B --fuse 8 --raster-group 4 > $O/f8_g4_$i.json 2>&1
  timeout 300 $B --fuse 3 --raster-group 10 > $O/f3_g10_$i.json 2>&1
done
timeout 300 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:update_acc -s 4 -c 2 --csv --log-file $O/ncu_f4_g8.csv python bench.py --steps 1 --warmup 1 --no-hetero --no-cpu-baseline --e2e-steps 0 --no-sample --fuse 4 --raster-group 8 > /dev/null 2>&1
