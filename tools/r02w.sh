O=gpurun_out/r02w; mkdir -p $O
for i in 1 2; do
  for sb in 1 0; do
    timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 --share-b $sb > $O/bench_sb${sb}_$i.json 2> $O/bench_sb${sb}_$i.err
  done
done
