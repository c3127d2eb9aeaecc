"""Probe: where in-kernel staging pays.  One device (optionally an SM cap in a
green partition), p = 1, b = 512 (K = 2048 per update), resident pmm_compute
with fused_staging 0 (standalone staging between updates) and 2 (forced
in-kernel); prints the k-loop times as JSON lines."""
import json
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

b = 512
cases = [(16, 4096), (16, 8192), (32, 6144), (32, 8192), (32, 12288), (64, 8192), (64, 12288), (64, 16384),
         (148, 8192), (148, 16384), (148, 24576)]
for cap, N in cases:
    n = N // b
    row = {"cap": cap, "N": N}
    for fs in (0, 2):
        caps = None if cap == 148 else [cap]
        with pkg.Context.local([0], sm_caps=caps) as ctx:
            if caps:
                ctx.set_option("sm_partition", 1)
            ctx.set_option("fused_staging", fs)
            ctx.setup(N, b, pkg.colpart_arrange(n, [n * n]), pkg.FPM_F32)
            ctx.fill_synthetic(1, 2, pkg.FPM_DIST_PM1)
            ts = []
            for _ in range(4):
                ts.append(ctx.compute().t_compute_s)
            row[f"t_fs{fs}"] = min(ts[1:])
    row["gain_pct"] = 100.0 * (row["t_fs0"] / row["t_fs2"] - 1.0)
    print(json.dumps(row), flush=True)
