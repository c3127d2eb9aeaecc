O=gpurun_out/r02v18; mkdir -p $O
for fs in 1 0; do
timeout 900 python studies/hetero.py --sm-partition 1 --graph 0 --refine 3 --insitu 1 --reps 3 --option share_b=1 --option fused_staging=$fs --out $O/hetero_fs$fs.json > $O/hetero_fs$fs.log 2>&1
done
timeout 900 python bench.py > $O/bench.json 2> $O/bench.err
