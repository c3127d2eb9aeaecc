O=gpurun_out/r02re6; mkdir -p $O
INTO=1 timeout 600 python studies/probes/e2e_timeline.py > $O/tl_default.jsonl 2> $O/tl_default.err
for L in 4 6 12; do timeout 600 python studies/probes/e2e_timeline.py e2e_tail=$L > $O/tl_L$L.jsonl 2> $O/tl_L$L.err; done
timeout 600 python studies/probes/e2e_timeline.py tail_band=4096 > $O/tl_band4096.jsonl 2> $O/tl_band4096.err
