O=gpurun_out/r02v16; mkdir -p $O
timeout 1200 python studies/probes/fs_crossover.py > $O/fs_crossover.jsonl 2> $O/fs_crossover.err
