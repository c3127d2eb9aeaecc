set -x
mkdir -p gpurun_out/r02b
lscpu > gpurun_out/r02b/lscpu.txt; nproc >> gpurun_out/r02b/lscpu.txt
timeout 1200 python -m pytest tests/test_gpu_fp32class.py tests/test_gpu_cpu_devices.py tests/test_gpu_tail.py -q -p no:cacheprovider -x > gpurun_out/r02b/pytest_focus.log 2>&1
echo "rc=$?" >> gpurun_out/r02b/pytest_focus.log
for CK in 512 256 1024 2048; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0 --chunk-k $CK > gpurun_out/r02b/bench_ck$CK.json 2>&1
done
timeout 300 python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0 --kernel-variant 8 > gpurun_out/r02b/bench_v8.json 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0 --kernel-variant 4 > gpurun_out/r02b/bench_v4.json 2>&1
