O=gpurun_out/r02re20; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_pmm.py -m gpu -q -p no:cacheprovider -k "sample" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
