O=gpurun_out/r02v7; mkdir -p $O
timeout 300 python studies/probes/coresidence.py > $O/coresidence.json 2> $O/coresidence.err
