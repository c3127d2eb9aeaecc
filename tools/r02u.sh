O=gpurun_out/r02u; mkdir -p $O
for i in 1 2 3; do
  timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > $O/bench_$i.json 2> $O/bench_$i.err
done
