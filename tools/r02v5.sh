O=gpurun_out/r02v5; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_pmm.py -q -p no:cacheprovider -k "group_times or span" > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 300 python studies/probes/kloop_timeline.py > $O/tl_default.json 2> $O/tl_default.err
timeout 300 python studies/probes/kloop_timeline.py graph=0 > $O/tl_nograph.json 2> $O/tl_nograph.err
