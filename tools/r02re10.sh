O=gpurun_out/r02re10; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_fp32class.py -m gpu -q -p no:cacheprovider -k multicast -x > $O/pytest_mc.log 2>&1; echo "rc=$?" >> $O/pytest_mc.log
grep -q "rc=0" $O/pytest_mc.log || exit 0
for i in 1 2; do
for v in -1 12 13; do
timeout 600 python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0 --kernel-variant $v > $O/bench_v${v}_$i.json 2> $O/bench_v${v}_$i.err
done; done
