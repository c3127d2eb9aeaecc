O=gpurun_out/r02v9; mkdir -p $O
export PADS=1 BLOCKS=128
for v in -1 4 2; do for c in -1 100 0; do
VARIANT=$v CARVEOUT=$c timeout 120 python studies/probes/coresidence2.py >> $O/cores3.jsonl 2>> $O/cores3.err
done; done
