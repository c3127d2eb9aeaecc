"""Probe: the timeline of one end-to-end pmm_run at c5 (host-streamed inputs,
band-streamed tail) next to the resident k-loop: per update group the staging
and update intervals (pmm_group_times), the upload / download times and the
host wall clock.  One JSON line per mode; the per-group table on stderr.
Usage: python studies/probes/e2e_timeline.py [option=value ...]"""
import json
import os
import sys
import time

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import torch  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

N = int(os.environ.get("N", "49152"))
b = int(os.environ.get("B", "1024"))
opts = dict(kv.split("=") for kv in sys.argv[1:])
n = N // b
rects = [(0, 0, 0, n, n)]


def report(mode, st, tl, wall=None):
    gaps = [tl[0][2]] + [tl[g][2] - tl[g - 1][3] for g in range(1, len(tl))]
    for g, (p0, p1, u0, u1) in enumerate(tl):
        print(f"{mode} g{g:2d} stage {1e3 * p0:8.3f}-{1e3 * p1:8.3f}  update {1e3 * u0:8.3f}-{1e3 * u1:8.3f} "
              f"({1e3 * (u1 - u0):7.3f} ms)  gap {1e3 * gaps[g]:6.3f} ms", file=sys.stderr)
    rec = {"mode": mode, "t_compute_s": st.t_compute_s, "t_upload_s": st.t_upload_s,
           "t_download_s": st.t_download_s, "updates_s": sum(u1 - u0 for _, _, u0, u1 in tl),
           "gaps_s": sum(gaps), "first_gap_s": gaps[0], "after_last_update_s": st.t_compute_s - tl[-1][3],
           "groups": len(tl), "timeline": tl}
    if wall is not None:
        rec["wall_s"] = wall
        rec["tflops_wall"] = 2 * N ** 3 / wall / 1e12
    print(json.dumps(rec), flush=True)


hA = torch.empty((N, N), dtype=torch.float32, pin_memory=True)
hB = torch.empty((N, N), dtype=torch.float32, pin_memory=True)
hC = torch.empty((N, N), dtype=torch.float32, pin_memory=True)
tmp = torch.empty((N, N), dtype=torch.float32, device="cuda")
pkg.k_fill_synthetic(tmp, pkg.FPM_F32, N, 5, N, 0, 0, N, N)
hA.copy_(tmp)
pkg.k_fill_synthetic(tmp, pkg.FPM_F32, N, 6, N, 0, 0, N, N)
hB.copy_(tmp)
del tmp
torch.cuda.empty_cache()
with pkg.Context.local([0]) as ctx:
    for k, v in opts.items():
        ctx.set_option(k, int(v))
    ctx.setup(N, b, rects, pkg.FPM_F32)
    ctx.fill_synthetic(5, 6, pkg.FPM_DIST_PM1)
    for _ in range(2):
        ctx.compute()
    st = ctx.compute()
    report("resident", st, ctx.group_times(0))
    if os.environ.get("INTO"):   # resident inputs, C copied out under a fused (not streamed) tail
        ctx.upload(hA, hB, N, 0, 0)
        for i in range(3):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            st = ctx.compute_into(hC, N, 0, 0)
            w = time.perf_counter() - t0
        report("compute_into", st, ctx.group_times(0), w)
    for i in range(3):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        st = ctx.run(hA, hB, hC, N, b, rects, pkg.FPM_F32)
        w = time.perf_counter() - t0
    report("pmm_run", st, ctx.group_times(0), w)
