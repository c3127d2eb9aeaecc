O=gpurun_out/r02y; mkdir -p $O
B="python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0"
for i in 1 2 3; do
  timeout 300 $B > $O/base_$i.json 2>&1
  timeout 300 $B --l2-hint-b 1 > $O/h1_$i.json 2>&1
  timeout 300 $B --chunk-k 1024 > $O/ck1024_$i.json 2>&1
  timeout 300 $B --raster-snake 1 --l2-hint-b 1 > $O/s1h1_$i.json 2>&1
done
