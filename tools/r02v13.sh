O=gpurun_out/r02v13; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_pmm.py -q -p no:cacheprovider -x -k "fused_staging or group_times" > $O/pytest_fs.log 2>&1; echo "rc=$?" >> $O/pytest_fs.log
timeout 900 python -m pytest tests/test_gpu_ipc.py -q -p no:cacheprovider -x > $O/pytest_ipc.log 2>&1; echo "rc=$?" >> $O/pytest_ipc.log
B="python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline"
for i in 1 2; do
timeout 400 $B > $O/fs1_$i.json 2>/dev/null
timeout 400 $B --fused-staging 0 > $O/fs0_$i.json 2>/dev/null
done
