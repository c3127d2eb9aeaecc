set -x
O=gpurun_out/r02e; mkdir -p $O
timeout 900 python studies/hetero.py --sm-partition 1 --graph 0 --refine 3 --insitu 1 --out $O/hetero_c4_r02_green_refine.json > $O/hetero.log 2>&1
timeout 1500 python studies/memcap.py --refine 4 --out $O/memcap_fig7_r02_sockets_refine.json > $O/memcap_sockets.log 2>&1
timeout 1500 python studies/memcap.py --refine 4 --caps 74,36,2,2,2,2,2,2,2,2,2,2,2,2,2,2 --names G1,G2,c0,c1,c2,c3,c4,c5,c6,c7,c8,c9,c10,c11,c12,c13 --c-caps-mib 1024,512,0,0,0,0,0,0,0,0,0,0,0,0,0,0 --out $O/memcap_fig7_r02_cores_refine.json > $O/memcap_cores.log 2>&1
