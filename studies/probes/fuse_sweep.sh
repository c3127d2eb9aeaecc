# c5 bench at several pivot-fusion depths (K = f * b per update launch), same box.
mkdir -p gpurun_out/fuse
for f in 2 4 3 6 2 4; do
  timeout 400 python bench.py --fuse $f --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample --steps 5 --warmup 3 \
    > gpurun_out/fuse/f$f.json 2> gpurun_out/fuse/f$f.err
  python - "$f" <<'PY'
import json,sys
f=sys.argv[1]
d=json.loads(open(f"gpurun_out/fuse/f{f}.json").read().strip().splitlines()[-1])
print("fuse",f,"value",round(d["value"]/1e3,1),"frac",round(d["roofline"]["frac"],4),"clk",d["clocks"]["sm_mhz"],d["clocks"].get("power_w_median"))
PY
done 2>&1 | tee gpurun_out/fuse/summary.txt
