O=gpurun_out/r02re14; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_bench_multi.py -m gpu -q -p no:cacheprovider > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
TR="python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1"
timeout 900 $TR --nproc-per-node 2 --master-port 29551 bench.py --gpus 2 --steps 3 --warmup 3 --same-gpu > $O/c5_x2.json 2> $O/c5_x2.err
