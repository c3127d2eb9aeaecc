O=gpurun_out/r02v17; mkdir -p $O
timeout 1200 python studies/probes/fs_crossover.py > $O/fs_crossover.jsonl 2> $O/fs_crossover.err
timeout 900 python -m pytest tests/test_gpu_pmm.py tests/test_gpu_green.py tests/test_gpu_ipc.py -q -p no:cacheprovider -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
