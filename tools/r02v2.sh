O=gpurun_out/r02v2; mkdir -p $O
timeout 120 ./studies/probes/nvls_probe > $O/nvls_probe.json 2>&1
