O=gpurun_out/r02re3; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_tail.py tests/test_gpu_pmm.py -m gpu -q -p no:cacheprovider > $O/pytest_tail_pmm.log 2>&1; echo "rc=$?" >> $O/pytest_tail_pmm.log
for i in 1 2; do
timeout 600 python bench.py --config c3 --no-hetero --steps 10 > $O/c3_auto_$i.json 2> $O/c3_auto_$i.err
timeout 600 python bench.py --config c3 --no-hetero --steps 10 --e2e-tail 1 > $O/c3_tail1_$i.json 2> $O/c3_tail1_$i.err
done
