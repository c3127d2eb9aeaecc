O=gpurun_out/r02v8; mkdir -p $O
timeout 300 python studies/probes/coresidence2.py > $O/cores2.json 2> $O/cores2.err
cuobjdump -res-usage studies/probes/libcoprobe.so > $O/coprobe_res.txt 2>&1
