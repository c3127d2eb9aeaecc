O=gpurun_out/r02re17; mkdir -p $O
B="python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0"
for i in 1 2 3; do
timeout 600 $B > $O/def_$i.json 2> /dev/null
timeout 600 $B --l2-hint-b 2 > $O/hintb2_$i.json 2> /dev/null
done
