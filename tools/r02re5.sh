O=gpurun_out/r02re5; mkdir -p $O
timeout 600 python studies/probes/e2e_timeline.py > $O/e2e_timeline.jsonl 2> $O/e2e_timeline.err
