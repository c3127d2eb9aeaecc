O=gpurun_out/r02re15; mkdir -p $O
for i in 1 2; do for v in -1 7; do
timeout 600 python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0 --kernel-variant $v > $O/v${v}_$i.json 2> $O/v${v}_$i.err
done; done
