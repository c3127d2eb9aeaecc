O=gpurun_out/r02v10; mkdir -p $O
PADS=1,48 BLOCKS=32,128,256 timeout 120 python studies/probes/coresidence2.py > $O/cores.json 2> $O/cores.err
timeout 300 python studies/probes/coresidence.py > $O/coresidence.json 2> $O/coresidence.err
timeout 300 python studies/probes/kloop_timeline.py > $O/tl_default.json 2> $O/tl_default.err
timeout 1200 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_f16i8.py tests/test_gpu_fp32class.py tests/test_gpu_pmm.py -q -p no:cacheprovider -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
timeout 600 python bench.py --steps 10 --warmup 3 --no-hetero > $O/bench.json 2> $O/bench.err
