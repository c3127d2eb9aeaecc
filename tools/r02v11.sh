O=gpurun_out/r02v11; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_pmm.py -q -p no:cacheprovider -x -k "fused_staging or group_times" > $O/pytest_fs.log 2>&1; echo "rc=$?" >> $O/pytest_fs.log
timeout 600 python -m pytest tests/test_gpu_ipc.py -q -p no:cacheprovider -x > $O/pytest_ipc.log 2>&1; echo "rc=$?" >> $O/pytest_ipc.log
timeout 300 python studies/probes/kloop_timeline.py > $O/tl_default.json 2> $O/tl_default.err
timeout 300 python studies/probes/kloop_timeline.py fused_staging=0 > $O/tl_off.json 2> $O/tl_off.err
