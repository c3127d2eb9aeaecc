mkdir -p gpurun_out/hyb
timeout 600 ncu --set full --clock-control none -k regex:"update_kernel|update_hyb_kernel" --launch-skip 1 --launch-count 3 -o gpurun_out/hyb/upd_full python studies/probes/hyb_one.py 16384 2048 > gpurun_out/hyb/ncu.log 2>&1
ls -la gpurun_out/hyb
