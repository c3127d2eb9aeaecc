O=gpurun_out/r02re13; mkdir -p $O
for i in 1 2; do
timeout 2000 python -m pytest tests -m gpu -q -p no:cacheprovider > $O/pytest_$i.log 2>&1; echo "rc=$?" >> $O/pytest_$i.log
done
