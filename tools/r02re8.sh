O=gpurun_out/r02re8; mkdir -p $O
timeout 1500 python -m pytest tests/test_gpu_pmm.py tests/test_gpu_ipc.py tests/test_gpu_green.py tests/test_gpu_tail.py -m gpu -q -p no:cacheprovider > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
