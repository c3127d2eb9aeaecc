O=gpurun_out/r02v15; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_pmm.py tests/test_gpu_green.py tests/test_gpu_ipc.py -q -p no:cacheprovider -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
for fs in 0 2; do
timeout 900 python studies/hetero.py --sm-partition 1 --graph 0 --refine 3 --insitu 1 --reps 3 --option share_b=1 --option fused_staging=$fs --out $O/hetero_fs$fs.json > $O/hetero_fs$fs.log 2>&1
done
