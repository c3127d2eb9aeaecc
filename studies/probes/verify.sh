# One GPU pass over the current tree: gpu tests, smoke, default bench line.
mkdir -p gpurun_out/verify
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit --format=csv > gpurun_out/verify/gpu.txt 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/verify/pytest_gpu.log 2>&1; echo "pytest exit $?" >> gpurun_out/verify/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/verify/smoke.log 2>&1; echo "smoke exit $?" >> gpurun_out/verify/smoke.log
timeout 900 python bench.py > gpurun_out/verify/bench.json 2> gpurun_out/verify/bench.err; echo "bench exit $?" >> gpurun_out/verify/bench.err
tail -3 gpurun_out/verify/pytest_gpu.log gpurun_out/verify/smoke.log; cat gpurun_out/verify/bench.json | head -c 600
