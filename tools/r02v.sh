O=gpurun_out/r02v; mkdir -p $O
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest.log 2>&1
echo "rc=$?" >> $O/pytest.log
timeout 900 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > $O/bench.json 2> $O/bench.err
timeout 900 python studies/scaling_emulated.py --out $O/scaling.json > $O/scaling.log 2>&1
