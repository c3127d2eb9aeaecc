O=gpurun_out/r02re11; mkdir -p $O
for i in 1 2; do
for cfg in "1 1" "2 0" "2 1" "1 0"; do set -- $cfg
timeout 600 python bench.py --steps 2 --warmup 3 --e2e-steps 0 --no-cpu-baseline --hetero-fused-staging $1 --share-b $2 > $O/h_fs$1_sb$2_$i.json 2> $O/h_fs$1_sb$2_$i.err
done; done
