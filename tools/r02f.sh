set -x
O=gpurun_out/r02f; mkdir -p $O
timeout 600 python bench.py --config c3 --steps 10 --warmup 3 --no-hetero > $O/bench_c3.json 2> $O/bench_c3.err
timeout 900 python bench.py --config c4 --steps 5 --warmup 3 > $O/bench_c4.json 2> $O/bench_c4.err
timeout 600 compute-sanitizer --tool memcheck python tools/sanitize_r02.py > $O/san_memcheck.log 2>&1
timeout 900 compute-sanitizer --tool racecheck python tools/sanitize_r02.py > $O/san_racecheck.log 2>&1
timeout 900 compute-sanitizer --tool synccheck python tools/sanitize_r02.py > $O/san_synccheck.log 2>&1
timeout 900 python studies/hybrid.py --out $O/hybrid_r02.json > $O/hybrid.log 2>&1
timeout 900 python studies/speed_sweep.py --out $O/speed_sweep_r02_f16x3.json > $O/speed_sweep.log 2>&1
for RG in 2 4 8; do
  timeout 900 python studies/hetero.py --sm-partition 1 --graph 0 --insitu 0 --option raster_group=$RG --out $O/hetero_rg$RG.json > $O/hetero_rg$RG.log 2>&1
done
timeout 1500 python studies/memcap.py --cliff 1 --refine 3 --arrange fpm --out $O/memcap_fig7_r02_sockets_cliff_level.json > $O/memcap_sockets.log 2>&1
timeout 900 python studies/hetero.py --sm-partition 1 --graph 0 --refine 3 --insitu 1 --out $O/hetero_c4_r02_green_level.json > $O/hetero_level.log 2>&1
