O=gpurun_out/r02v3; mkdir -p $O
timeout 120 ./studies/probes/nvls_probe > $O/nvls_probe.json 2>&1
