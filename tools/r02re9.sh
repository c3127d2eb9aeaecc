O=gpurun_out/r02re9; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_ipc.py tests/test_gpu_bench_multi.py -m gpu -q -p no:cacheprovider > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
