mkdir -p gpurun_out/ts
for L in ${TAILS:--1 7 8 9 10 11 12}; do
  timeout 400 python bench.py --no-hetero --no-cpu-baseline --no-sample --steps 1 --warmup 3 --e2e-steps 3 --e2e-tail $L > gpurun_out/ts/L.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/ts/L.json').read().strip().splitlines()[-1]); print('e2e_tail', $L, 'value', round(d['value']/1e3,1), 'e2e', round(d['e2e']['value']/1e3,1), d['e2e']['ms_per_step'], d['e2e']['download_s'], d['e2e']['device_kloop_s'])"
done
D=gpurun_out/r01e; mkdir -p $D
timeout 600 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:update_hyb_kernel --csv --log-file $D/update_traffic.csv python bench.py --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample --steps 1 --warmup 0 > $D/traffic_bench.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_hyb_kernel --launch-skip 30 --launch-count 1 -o $D/update_full python bench.py --steps 1 --warmup 2 --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample > $D/full_bench.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file $D/launches.csv python bench.py --no-hetero --e2e-steps 0 --no-cpu-baseline --no-sample --steps 1 --warmup 3 > $D/launches_bench.log 2>&1
ls $D
