O=gpurun_out/r02r; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_cpu_devices.py tests/test_gpu_pmm.py -q -p no:cacheprovider -k "synchronised or sample or mixed" > $O/pytest.log 2>&1
echo "rc=$?" >> $O/pytest.log
timeout 1200 python studies/hybrid.py --refine 3 --out $O/hybrid_r02_sync.json > $O/hybrid.log 2>&1
timeout 1200 python studies/hybrid.py --sockets 15 --refine 3 --out $O/hybrid_r02_one_socket_sync.json > $O/hybrid1.log 2>&1
