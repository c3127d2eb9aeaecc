O=gpurun_out/r02m; mkdir -p $O
timeout 900 python bench.py --steps 10 --warmup 3 > $O/bench.json 2> $O/bench.err
timeout 900 python bench.py --config c4 --steps 5 --warmup 3 > $O/bench_c4.json 2> $O/bench_c4.err
timeout 900 python -m pytest tests/test_gpu_bench_multi.py tests/test_bench_contract.py -q -p no:cacheprovider > $O/pytest.log 2>&1
echo "rc=$?" >> $O/pytest.log
