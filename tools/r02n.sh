O=gpurun_out/r02n; mkdir -p $O
timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 --same-gpu > $O/bench_n2_samegpu.json 2> $O/bench_n2_samegpu.err
echo "rc=$?" >> $O/bench_n2_samegpu.err
timeout 1200 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29512 bench.py --gpus 4 --steps 3 --warmup 3 --same-gpu --config c3 > $O/bench_n4_c3_samegpu.json 2> $O/bench_n4_c3_samegpu.err
echo "rc=$?" >> $O/bench_n4_c3_samegpu.err
