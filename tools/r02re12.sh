O=gpurun_out/r02re12; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_tail.py -m gpu -q -p no:cacheprovider > $O/pytest_tail.log 2>&1; echo "rc=$?" >> $O/pytest_tail.log
for i in 1 2 3; do for r in 0 1; do
timeout 600 python bench.py --steps 3 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 5 --tail-ramp $r > $O/ramp${r}_$i.json 2> $O/ramp${r}_$i.err
done; done
