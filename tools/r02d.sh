set -x
O=gpurun_out/r02d; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_ipc.py tests/test_gpu_bench_multi.py -q -p no:cacheprovider > $O/pytest_ipc_multi.log 2>&1
echo "rc=$?" >> $O/pytest_ipc_multi.log
for F in 4 8; do
  timeout 300 python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0 --fuse $F > $O/bench_f$F.json 2>&1
done
timeout 300 python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0 --fuse 4 --chunk-k 1024 > $O/bench_f4_ck1024.json 2>&1
timeout 600 python studies/contention.py --out $O/contention_r02.json > $O/contention.log 2>&1
