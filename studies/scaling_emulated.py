#!/usr/bin/env python
"""Strong scaling of config 5 emulated on ONE B200 (SURVEY §8(d) c5 "strong
scaling 1 -> 8 GPUs", §8(e)): p = 1, 2, 4, 8 devices, each a disjoint
green-context partition of floor(148 / p) SMs (even), homogeneous FPM partition
and column arrangement of N = 49152, b = 1024, the same k-loop (pivot exchange
fused into staging, rank-(f b) updates) as on p GPUs.

With one GPU the aggregate tensor throughput is fixed, so a flat line is the
ideal: what drops with p is the method's own overhead -- the exchange and
staging the partition adds (each device stages (h_i + w_i) b^2 per pivot,
P:15), the arrangement's rounding imbalance, the smaller per-device problems.
Reported per p: TFLOP/s, measured imbalance, pivot bytes moved, the share of
staging hidden under the updates.  Writes JSON (profiles/scaling_emulated_r02.json).
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402


def imbalance(ts):
    live = [t for t in ts if t > 0]
    return max(live) / (sum(live) / len(live)) - 1.0 if live else 0.0


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--N", type=int, default=49152)
    ap.add_argument("--b", type=int, default=1024)
    ap.add_argument("--ps", default="1,2,4,8")
    ap.add_argument("--reps", type=int, default=3)
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "scaling_emulated_r02.json"))
    args = ap.parse_args()
    N, b = args.N, args.b
    n = N // b
    rows = []
    for p in [int(x) for x in args.ps.split(",")]:
        cap = (148 // p) // 2 * 2
        devs = [0] * p
        ctx = pkg.Context.local(devs, sm_caps=[cap] * p if p > 1 else None)
        if p > 1:
            ctx.set_option("sm_partition", 1)
        d = pkg.fpm_partition(n * n, [([1], [1.0])] * p)
        rects = pkg.colpart_arrange_fpm(n, d, [([1], [1.0])] * p)
        ctx.setup(N, b, rects, pkg.FPM_F32)
        ctx.fill_synthetic(5, 6, pkg.FPM_DIST_PM1)
        ctx.compute()
        best = None
        for _ in range(args.reps):
            st = ctx.compute()
            if best is None or st.t_compute_s < best.t_compute_s:
                best = st
        comp = list(best.per_dev_compute_s[:p])
        upd = list(best.per_dev_update_s[:p])
        stage = [c - u for c, u in zip(comp, upd)]
        rows.append({"p": p, "sm_cap": cap if p > 1 else 148, "rects": rects, "t_s": best.t_compute_s,
                     "tflops": best.gflops / 1e3, "imbalance": imbalance(comp), "comm_bytes": best.comm_bytes,
                     "per_dev_compute_s": comp, "per_dev_update_s": upd,
                     "staging_share_of_compute": sum(stage) / sum(comp),
                     "exposed_s": best.t_compute_s - max(upd)})
        print(f"p={p} cap={cap}: {best.gflops / 1e3:7.1f} TFLOP/s  imb={100 * imbalance(comp):5.2f}%  "
              f"comm={best.comm_bytes / 1e9:7.2f} GB  staging share={100 * rows[-1]['staging_share_of_compute']:.1f}%",
              flush=True)
        ctx.close()
    out = {"config": {"N": N, "b": b, "dtype": "f32 (F16X3)", "partition": "homogeneous, FPM-chosen integers",
                      "devices": "green-context partitions of one B200"}, "rows": rows}
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
