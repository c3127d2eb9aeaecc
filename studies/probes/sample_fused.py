"""Probe: fpm_sample with the update's in-kernel staging (the k-loop's path
where it applies) against the standalone split + update (fused_staging = 0),
one device alone on the GPU and capped devices, b = 512, and the per-group
time of the resident k-loop at the same rectangle for reference."""
import json
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

b = 512
ms = [8, 12, 16, 24, 32]
out = []
for cap in (0, 64, 32):
    row = {"sm_cap": cap}
    for fs in (0, 1):
        with pkg.Context.local([0], sm_caps=[cap] if cap else None) as ctx:
            ctx.set_option("fused_staging", fs)
            sp, ci, reps = ctx.sample(0, b, [m * m for m in ms], pkg.FPM_F32)
            row[f"fs{fs}"] = [s / 1e12 for s in sp]
    # the k-loop: group time of a p = 1 problem of side m b (resident, default options)
    kl = []
    for m in ms:
        N = m * b
        with pkg.Context.local([0], sm_caps=[cap] if cap else None) as ctx:
            ctx.setup(N, b, pkg.colpart_arrange(m, [m * m]), pkg.FPM_F32)
            ctx.fill_synthetic(1, 2)
            for _ in range(2):
                ctx.compute()
            st = ctx.compute()
            kl.append(2.0 * N ** 3 / st.t_compute_s / 1e12)
    row["kloop"] = kl
    row["m"] = ms
    out.append(row)
    print(json.dumps(row), flush=True)
