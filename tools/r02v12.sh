O=gpurun_out/r02v12; mkdir -p $O
B="python bench.py --steps 8 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0"
for i in 1 2; do
timeout 300 $B > $O/fs1_$i.json 2>/dev/null
FPM_FS=0 timeout 300 $B --fused-staging 0 > $O/fs0_$i.json 2>/dev/null
done
timeout 900 python -m pytest tests/test_gpu_pmm.py -q -p no:cacheprovider -x -k "fused_staging or group_times" > $O/pytest_fs.log 2>&1; echo "rc=$?" >> $O/pytest_fs.log
