O=gpurun_out/r02aa; mkdir -p $O
B="python bench.py --steps 2 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 5"
for i in 1 2; do
  timeout 600 $B > $O/base_$i.json 2>&1
  timeout 600 $B --tail-band 1024 > $O/tb1024_$i.json 2>&1
  timeout 600 $B --tail-band 4096 > $O/tb4096_$i.json 2>&1
  timeout 600 $B --e2e-tail 14 > $O/t14_$i.json 2>&1
  timeout 600 $B --e2e-tail 10 > $O/t10_$i.json 2>&1
done
