O=gpurun_out/r02x; mkdir -p $O
timeout 1800 python studies/memcap.py --cliff 1 --refine 3 --arrange fpm --out $O/memcap_fig7_r02_sockets.json > $O/memcap_sockets.log 2>&1
timeout 2400 python studies/memcap.py --cliff 1 --refine 3 --arrange fpm --caps 74,36,2,2,2,2,2,2,2,2,2,2,2,2,2,2 --names G1,G2,c0,c1,c2,c3,c4,c5,c6,c7,c8,c9,c10,c11,c12,c13 --c-caps-mib 1024,512,0,0,0,0,0,0,0,0,0,0,0,0,0,0 --out $O/memcap_fig7_r02_cores.json > $O/memcap_cores.log 2>&1
