mkdir -p gpurun_out/studies6
timeout 900 python bench.py > gpurun_out/studies6/bench.json 2> gpurun_out/studies6/bench.err
timeout 900 python studies/speed_sweep.py --out gpurun_out/studies6/speed_sweep_r01_f16i8.json > gpurun_out/studies6/speed_sweep.log 2>&1
timeout 900 python studies/hetero.py --out gpurun_out/studies6/hetero_c4_r01_f16i8.json > gpurun_out/studies6/hetero.log 2>&1
timeout 900 python studies/hetero.py --sm-partition 1 --out gpurun_out/studies6/hetero_c4_r01_f16i8_green.json > gpurun_out/studies6/hetero_green.log 2>&1
timeout 900 python studies/configs.py gpurun_out/studies6/configs_r01_f16i8.json > gpurun_out/studies6/configs.log 2>&1
tail -3 gpurun_out/studies6/configs.log
