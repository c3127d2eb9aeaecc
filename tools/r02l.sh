O=gpurun_out/r02l; mkdir -p $O
B="--steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0"
for i in 1 2 3; do
  (cd tmp_old && timeout 300 python bench.py $B > ../$O/old_$i.json 2>&1)
  timeout 300 python bench.py $B > $O/new_$i.json 2>&1
done
