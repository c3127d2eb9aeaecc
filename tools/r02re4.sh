O=gpurun_out/r02re4; mkdir -p $O
TR="python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1"
NCCL_DEBUG=WARN timeout 300 $TR --nproc-per-node 2 --master-port 29541 bench.py --gpus 2 --same-gpu --transport nccl --config c3 --N 4096 --steps 2 --warmup 3 --no-hetero --no-cpu-baseline > $O/nccl2_samegpu.json 2> $O/nccl2_samegpu.err; echo "rc=$?" >> $O/nccl2_samegpu.err
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; echo "rc=$?" >> $O/smoke.log
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
