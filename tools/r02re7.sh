O=gpurun_out/r02re7; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_fp32class.py -m gpu -q -p no:cacheprovider -k e2e_full > $O/pytest_e2e_full.log 2>&1; echo "rc=$?" >> $O/pytest_e2e_full.log
