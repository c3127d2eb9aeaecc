set -x
mkdir -p gpurun_out/r02a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > gpurun_out/r02a/smi.txt
timeout 900 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/r02a/pytest.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r02a/pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/r02a/bench.json 2> gpurun_out/r02a/bench.err
for G in 16 24 32 48; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0 --raster-group $G > gpurun_out/r02a/bench_G$G.json 2>&1
done
