set -x
O=gpurun_out/r02i; mkdir -p $O
timeout 900 python -m pytest tests/test_gpu_fp32class.py -q -p no:cacheprovider -k "edge or tile_order or one_fused" > $O/pytest.log 2>&1
echo "rc=$?" >> $O/pytest.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1
echo "rc=$?" >> $O/smoke.log
