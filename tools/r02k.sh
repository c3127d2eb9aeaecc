set -x
O=gpurun_out/r02k; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_pmm.py -q -p no:cacheprovider -k "span or sample_rects or config1" > $O/pytest.log 2>&1
echo "rc=$?" >> $O/pytest.log
timeout 900 python studies/hybrid.py --sockets 15 --out $O/hybrid_r02_one_socket.json > $O/hybrid.log 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 > $O/bench.json 2> $O/bench.err
