# Round-1 studies rerun with the F16I8 default scheme.
mkdir -p gpurun_out/studies
timeout 300 python -m pytest tests/test_gpu_f16i8.py -x -q > gpurun_out/studies/pytest_f16i8.log 2>&1; tail -2 gpurun_out/studies/pytest_f16i8.log
timeout 900 python studies/speed_sweep.py --out gpurun_out/studies/speed_sweep_r01_f16i8.json > gpurun_out/studies/speed_sweep.log 2>&1; tail -3 gpurun_out/studies/speed_sweep.log
timeout 900 python studies/hetero.py --out gpurun_out/studies/hetero_c4_r01_f16i8.json > gpurun_out/studies/hetero.log 2>&1; tail -12 gpurun_out/studies/hetero.log
timeout 900 python studies/hetero.py --sm-partition 1 --out gpurun_out/studies/hetero_c4_r01_f16i8_green.json > gpurun_out/studies/hetero_green.log 2>&1; tail -12 gpurun_out/studies/hetero_green.log
timeout 900 python studies/configs.py gpurun_out/studies/configs_r01_f16i8.json > gpurun_out/studies/configs.log 2>&1; tail -12 gpurun_out/studies/configs.log
