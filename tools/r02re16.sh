O=gpurun_out/r02re16; mkdir -p $O
B="python bench.py --steps 5 --warmup 3 --no-hetero --no-cpu-baseline --e2e-steps 0"
for i in 1 2; do
timeout 600 $B > $O/def_$i.json 2> /dev/null
timeout 600 $B --raster-group 12 > $O/rg12_$i.json 2> /dev/null
timeout 600 $B --raster-group 20 > $O/rg20_$i.json 2> /dev/null
timeout 600 $B --chunk-k 1024 > $O/ck1024_$i.json 2> /dev/null
timeout 600 $B --l2-hint-b 1 > $O/hintb1_$i.json 2> /dev/null
done
