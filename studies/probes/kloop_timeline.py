"""Probe: where the c5 k-loop's time goes beyond its updates.  Runs the bench's
resident step (pmm_compute, default options) and prints, per update group, the
staging interval, the update interval and the gap before the update starts
(pmm_group_times); summary as one JSON line."""
import json
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

N = int(os.environ.get("N", "49152"))
b = int(os.environ.get("B", "1024"))
opts = dict(kv.split("=") for kv in sys.argv[1:])
n = N // b
with pkg.Context.local([0]) as ctx:
    for k, v in opts.items():
        ctx.set_option(k, int(v))
    ctx.setup(N, b, pkg.colpart_arrange(n, [n * n]), pkg.FPM_F32)
    ctx.fill_synthetic(1, 2, pkg.FPM_DIST_PM1)
    for _ in range(3):
        ctx.compute()
    st = ctx.compute()
    tl = ctx.group_times(0)
gaps = [tl[0][2]] + [tl[g][2] - tl[g - 1][3] for g in range(1, len(tl))]
late = [max(0.0, tl[g][1] - tl[g - 1][3]) for g in range(1, len(tl))]   # staging g ended after update g-1
for g, (p0, p1, u0, u1) in enumerate(tl):
    print(f"g{g:2d} stage {1e3 * p0:8.3f}-{1e3 * p1:8.3f}  update {1e3 * u0:8.3f}-{1e3 * u1:8.3f} "
          f"({1e3 * (u1 - u0):6.3f} ms)  gap {1e3 * gaps[g]:6.3f} ms", file=sys.stderr)
upd = sum(u1 - u0 for _, _, u0, u1 in tl)
print(json.dumps({"N": N, "b": b, "options": opts, "t_compute_s": st.t_compute_s, "updates_s": upd,
                  "gaps_s": sum(gaps), "first_gap_s": gaps[0], "tail_s": st.t_compute_s - tl[-1][3],
                  "staging_late_s": sum(late), "groups": len(tl),
                  "timeline": tl}))
