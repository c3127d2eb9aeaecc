O=gpurun_out/r02re18; mkdir -p $O
timeout 900 python studies/probes/sample_fused.py > $O/sample_fused.jsonl 2> $O/sample_fused.err
timeout 1500 python -m pytest tests/test_gpu_pmm.py tests/test_gpu_cpu_devices.py tests/test_gpu_green.py tests/test_gpu_ooc.py -m gpu -q -p no:cacheprovider > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
