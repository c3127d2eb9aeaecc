O=gpurun_out/r02re19; mkdir -p $O
TR="python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1"
timeout 1200 $TR --nproc-per-node 4 --master-port 29561 bench.py --gpus 4 --steps 3 --warmup 3 --same-gpu > $O/c5_x4.json 2> $O/c5_x4.err
timeout 1200 $TR --nproc-per-node 8 --master-port 29562 bench.py --gpus 8 --steps 3 --warmup 3 --same-gpu --config c3 > $O/c3_x8.json 2> $O/c3_x8.err
