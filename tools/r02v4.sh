O=gpurun_out/r02v4; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_bench_multi.py -q -p no:cacheprovider > $O/pytest_multi.log 2>&1; echo "rc=$?" >> $O/pytest_multi.log
TR="python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1"
timeout 900 $TR --nproc-per-node 2 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --same-gpu > $O/c5_x2.json 2> $O/c5_x2.err; echo "rc=$?" >> $O/c5_x2.err
timeout 900 $TR --nproc-per-node 4 --master-port 29512 bench.py --gpus 4 --steps 3 --warmup 3 --same-gpu --config c3 > $O/c3_x4.json 2> $O/c3_x4.err; echo "rc=$?" >> $O/c3_x4.err
