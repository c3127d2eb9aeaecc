"""Probe: where the end-to-end pmm_run time goes at c5 (N = 49152, b = 1024),
against the resident k-loop, for a few fuse settings.  Prints one JSON line per
variant.  Usage: python studies/probes/e2e_probe.py [--fuse 0 4] [--reps 2]"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))

import torch  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402


def stats_dict(st, wall=None):
    d = {"t_compute_s": st.t_compute_s, "t_upload_s": st.t_upload_s, "t_download_s": st.t_download_s,
         "update_s": st.per_dev_update_s[0], "compute_s": st.per_dev_compute_s[0], "updates": st.updates,
         "tflops_kloop": 2 * N ** 3 / st.t_compute_s / 1e12}
    if wall is not None:
        d["wall_s"] = wall
        d["tflops_wall"] = 2 * N ** 3 / wall / 1e12
    return d


ap = argparse.ArgumentParser()
ap.add_argument("--N", type=int, default=49152)
ap.add_argument("--b", type=int, default=1024)
ap.add_argument("--fuse", type=int, nargs="+", default=[0, 4])
ap.add_argument("--tail", type=int, nargs="+", default=[-1])
ap.add_argument("--band", type=int, nargs="+", default=[2048])
ap.add_argument("--tail-fuse", type=int, nargs="+", default=[1])
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--no-e2e", action="store_true")
args = ap.parse_args()
N, b = args.N, args.b
n = N // b
rects = [(0, 0, 0, n, n)]
ctx = pkg.Context.local([0])
ctx.setup(N, b, rects, pkg.FPM_F32)
ctx.fill_synthetic(5, 6, pkg.FPM_DIST_PM1)
hA = hB = hC = None
if not args.no_e2e:
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
for fuse in args.fuse:
    ctx.set_option("fuse", fuse)
    ctx.setup(N, b, rects, pkg.FPM_F32)
    ctx.fill_synthetic(5, 6, pkg.FPM_DIST_PM1)
    for _ in range(2):
        ctx.compute()
    res = [stats_dict(ctx.compute()) for _ in range(args.reps)]
    print(json.dumps({"fuse": fuse, "mode": "resident", "runs": res}), flush=True)
    if args.no_e2e:
        continue
    for tail, band, tf in [(t, bd, tf) for t in args.tail for bd in args.band for tf in args.tail_fuse]:
        ctx.set_option("e2e_tail", tail)
        ctx.set_option("tail_band", band)
        ctx.set_option("tail_fuse", tf)
        out = []
        for i in range(args.reps + 1):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            st = ctx.run(hA, hB, hC, N, b, rects, pkg.FPM_F32)
            w = time.perf_counter() - t0
            if i:
                out.append(stats_dict(st, w))
        print(json.dumps({"fuse": fuse, "tail": tail, "band": band, "tail_fuse": tf, "mode": "pmm_run", "runs": out}), flush=True)
ctx.close()
