# c5 bench (k-loop only) over fuse x kernel variant x raster group, same box.
mkdir -p gpurun_out/sweep
run() {  # name, extra args
  timeout 300 python bench.py --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample --steps 5 --warmup 3 $2 \
    > gpurun_out/sweep/$1.json 2> gpurun_out/sweep/$1.err
  python - "$1" <<'PY'
import json,sys
n=sys.argv[1]
try:
    d=json.loads(open(f"gpurun_out/sweep/{n}.json").read().strip().splitlines()[-1])
    print(n,"value",round(d["value"]/1e3,1),"upd",round(d["roofline"]["achieved"],1),"clk",d["clocks"]["sm_mhz"],d["clocks"].get("power_w_median"),flush=True)
except Exception as e:
    print(n,"FAILED",e,flush=True)
PY
}
# specs "name:args" from the command line (default: the round-1 sweep)
[ $# -gt 0 ] || set -- "base:" "f4:--fuse 4" "v0:--kernel-variant 0" "v1:--kernel-variant 1" "r32:--raster-group 32" \
  "r8:--raster-group 8" "f1:--fuse 1" "f3:--fuse 3" "hintB1:--l2-hint-b 1" "x3:--scheme f16x3" "base2:"
for spec in "$@"; do
  run "${spec%%:*}" "${spec#*:}"
done 2>&1 | tee gpurun_out/sweep/summary.txt
