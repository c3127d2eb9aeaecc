#!/usr/bin/env python
"""Memory-cliff study (Table III / Fig. 6 / Fig. 7 analogue, SURVEY §8(f)
NEXT-1 and NEXT-2) on ONE B200.

The paper's hybrid node: two GPUs whose device memory holds C_i only
up to some problem size (GTX680 "G1", C870 "G2"), beyond which their
out-of-core kernel (versions 2-3) streams C_i over PCIe and the speed
"drops" (Fig. 3); plus CPU sockets ("S5", "S6") with no such limit.  CPM
constants measured while the problem fits overload G1 once it no longer fits
("the CPM-based data partitioning results in overloading GeForce GTX680,
starting from matrix size 50x50"); FPM, whose speed functions include the
cliff, does not.

Emulation: six devices on one GPU, SM caps {74, 36, 8, 8, 8, 8} (G1 : S = 9.25,
the paper's "around 9 times"), per-device C caps (pmm_set_device_option
"c_cap_bytes") of 1 GiB for G1 and 0.5 GiB for G2 (none for the S devices), so
with b = 512 G1 holds up to 1024 blocks of C in core and G2 512.  Each device's
FPM is sampled with fpm_sample (which times out-of-core sizes out of core);
the multiply runs for n x n blocks, n in {40, 50, 60, 70}, under

  fpm   fpm_partition on the sampled speed functions
  cpm   constant models = each device's speed at the even share of the 40 x 40
        problem (constants "obtained in advance, from the speed
        measurements when some workload is distributed evenly") -- reading Q9
  homogeneous  equal areas ("data distributed evenly")

Fig. 7 is the total time per n and partition (exchange included);
Fig. 6 the per-device computation time at 60 x 60 (per_dev_compute_s).

Reported per n and partition (Table III's columns): blocks per device, total
time, per-device computation time, measured imbalance, whether each GPU ran out
of core.  Writes JSON (default profiles/memcap_table3_r01.json).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402


def imbalance(ts):
    live = [t for t in ts if t > 0]
    return max(live) / (sum(live) / len(live)) - 1.0 if live else 0.0


def pcie_bandwidth(nbytes=1 << 30, reps=5):
    """Pinned host <-> device copy bandwidth (GB/s): the out-of-core path's roofline."""
    import torch
    h = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    h2 = torch.empty(nbytes, dtype=torch.uint8).pin_memory()
    d = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    d2 = torch.empty(nbytes, dtype=torch.uint8, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()

    def timed(fn):
        best = float("inf")
        for _ in range(reps):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            fn()
            torch.cuda.synchronize()
            best = min(best, time.perf_counter() - t0)
        return best

    t_h2d = timed(lambda: d.copy_(h, non_blocking=True))
    t_d2h = timed(lambda: h.copy_(d, non_blocking=True))

    def both():
        with torch.cuda.stream(s1):
            d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2):
            h2.copy_(d2, non_blocking=True)
    t_bi = timed(both)
    return {"h2d_gbs": nbytes / t_h2d / 1e9, "d2h_gbs": nbytes / t_d2h / 1e9,
            "bidir_gbs": 2 * nbytes / t_bi / 1e9, "bytes": nbytes}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--b", type=int, default=512)
    ap.add_argument("--ns", default="30,40,45,50,55,60,65,70")
    ap.add_argument("--caps", default="74,36,8,8,8,8")
    ap.add_argument("--names", default="G1,G2,S1,S2,S3,S4")
    ap.add_argument("--c-caps-mib", default="1024,512,0,0,0,0")
    ap.add_argument("--ncal", type=int, default=40, help="CPM calibration problem, in blocks per side")
    ap.add_argument("--sizes", default="2,4,6,8,10,12,14,16,18,20,22,23,24,26,28,30,32,33,34,36,40,44,48,52,56")
    ap.add_argument("--cpu-sizes", default="2,4,8,12,16,20,24",
                    help="sample sides of CPU devices (their speed is flat beyond; the model is constant past the end)")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--ooc-keep", type=int, default=1)
    ap.add_argument("--ooc-buffers", type=int, default=2, help="R band buffers (2 = the paper's C0, C1)")
    ap.add_argument("--concurrent", action="store_true",
                    help="sample all devices at once (P:10 (ii)): the out-of-core GPUs then share the "
                         "host link as they do in the run")
    ap.add_argument("--link-group", default="",
                    help="comma-separated device indices sampled together in a context of their own "
                         "(the out-of-core GPUs: they share the host link in the run, P:10 (ii) applied to "
                         "the shared resource); the others alone")
    ap.add_argument("--sm-partition", type=int, default=0,
                    help="1 = each device in its own green-context SM partition (all its kernels confined)")
    ap.add_argument("--refine", type=int, default=0,
                    help="FPM: rounds of synchronised level correction (reading Q26): every device timed on the "
                         "rectangle it was given, all at once, its model rescaled, re-partition (fpm_refined)")
    ap.add_argument("--cliff", type=int, default=1,
                    help="1: bracket each capped GPU's memory cliff with two near-square samples (Q26)")
    ap.add_argument("--arrange", choices=["paper", "fpm"], default="paper",
                    help="FPM partition arranged by colpart_arrange (paper) or colpart_arrange_fpm (Q25)")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "memcap_table3_r01.json"))
    args = ap.parse_args()
    # "cpuN": a host-CPU device of N pinned cores (NEXT-3: the paper's sockets, P:18 s_c(x))
    cpu_dev = [c.startswith("cpu") for c in args.caps.split(",")]
    caps = [int(c[3:]) if c.startswith("cpu") else int(c) for c in args.caps.split(",")]
    names = args.names.split(",")
    c_caps = [int(c) << 20 for c in args.c_caps_mib.split(",")]
    p, b = len(caps), args.b
    ns = [int(x) for x in args.ns.split(",")]
    sizes = [int(m) ** 2 for m in args.sizes.split(",")]
    cpu_sizes = [int(m) ** 2 for m in args.cpu_sizes.split(",")]

    pcie = pcie_bandwidth()
    print("pcie", pcie, flush=True)
    def apply_options(c, devs):
        """Every option of the run on context c whose devices are `devs` (indices into caps)."""
        c.set_option("sm_partition", args.sm_partition)
        c.set_option("ooc_keep", args.ooc_keep)
        c.set_option("ooc_buffers", args.ooc_buffers)
        for j, i in enumerate(devs):
            if not cpu_dev[i]:
                c.set_device_option(j, "c_cap_bytes", c_caps[i])

    ctx = pkg.Context.local([pkg.FPM_CPU_DEVICE if c else 0 for c in cpu_dev], sm_caps=caps)
    apply_options(ctx, range(p))
    t0 = time.perf_counter()
    models, sample_info = [], []
    if args.concurrent:
        per_dev = list(zip(*ctx.sample(-1, b, sizes, pkg.FPM_F32)))
    else:                  # each device alone, as the paper measured its GPUs
        per_dev = [ctx.sample(dev, b, cpu_sizes if cpu_dev[dev] else sizes, pkg.FPM_F32) for dev in range(p)]
    if args.link_group:    # the link-sharing devices again, together in a context of their own
        grp = [int(i) for i in args.link_group.split(",")]
        with pkg.Context.local([0] * len(grp), sm_caps=[caps[i] for i in grp]) as gctx:
            apply_options(gctx, grp)
            gsp = list(zip(*gctx.sample(-1, b, sizes, pkg.FPM_F32)))
        for j, i in enumerate(grp):
            per_dev[i] = gsp[j]
    for dev, (sp, ci, reps) in enumerate(per_dev):
        models.append((cpu_sizes if cpu_dev[dev] else sizes, sp))
        sample_info.append({"name": names[dev], "sm_cap": None if cpu_dev[dev] else caps[dev],
                            "cpu_cores": caps[dev] if cpu_dev[dev] else None, "c_cap_bytes": c_caps[dev],
                            "speeds_gflops": [s / 1e9 for s in sp], "rel_ci95": ci, "reps": reps})
        print(f"{names[dev]}: " + " ".join(f"{m}:{s / 1e12:.1f}" for m, s in
                                           zip(args.sizes.split(","), sp)), flush=True)
    t_sample = time.perf_counter() - t0

    x_cal = max(1, args.ncal * args.ncal // p)
    cpm_models = [([1], [pkg.fpm_model_speed(m, x_cal)]) for m in models]

    def arrange(n, d, mods):
        return pkg.colpart_arrange_fpm(n, d, mods) if args.arrange == "fpm" else pkg.colpart_arrange(n, d)

    from studies import refine as rf
    splits, cliffs = [None] * p, [None] * p
    if args.cliff:   # bracket each capped GPU device's memory cliff with two samples (Q26)
        for i in range(p):
            if c_caps[i] and not cpu_dev[i]:
                models[i] = rf.cliff_points(ctx, i, b, models[i], c_caps[i])
                (x_in, r_in), (x_out, r_out) = rf.cliff_areas(c_caps[i], b)
                splits[i], cliffs[i] = x_in, (r_in, r_out)
                sample_info[i]["cliff_points"] = [(x, s / 1e9) for x, s in zip(*models[i])
                                                  if x not in sizes]

    table = []
    for n in ns:
        N, T = n * b, n * n
        row = {"n": n, "N": N}
        parts = [("fpm", models, None)]
        if args.refine:
            r_models, hist, r_d, r_rects = rf.refine(ctx, n, b, models, args.refine, arrange=args.arrange,
                                                      concurrent=True, splits=splits, cliffs=cliffs,
                                                      log=lambda m: print(m, flush=True))
            row["refine"] = hist
            parts.append(("fpm_refined", r_models, r_rects))
        parts += [("cpm", cpm_models, None), ("homogeneous", [([1], [1.0])] * p, None)]
        for name, mods, given in parts:
            d = pkg.fpm_partition(T, mods)
            rects = given if given is not None else (arrange(n, d, mods) if name == "fpm" else pkg.colpart_arrange(n, d))
            ctx.setup(N, b, rects, pkg.FPM_F32)
            ctx.fill_synthetic(5, 6, pkg.FPM_DIST_PM1)
            ctx.compute()
            best = None
            for _ in range(args.reps):
                st = ctx.compute()
                if best is None or st.t_compute_s < best.t_compute_s:
                    best = st
            areas = [r[3] * r[4] for r in rects]
            per_dev = list(best.per_dev_compute_s[:p])
            # FPM-predicted k-loop time: 2 a b^2 N flop at the model's speed s(a)
            pred = [2.0 * a * b * b * N / pkg.fpm_model_speed(m, a) if a > 0 else 0.0
                    for a, m in zip(areas, mods if name.startswith("fpm") else models)]
            row[name] = {
                "d": d, "areas": areas, "rects": rects,
                "t_total_s": best.t_compute_s, "gflops": best.gflops,
                "per_dev_compute_s": per_dev, "imbalance_measured": imbalance(per_dev),
                "fpm_predicted_time_s": max(pred),
                "ooc": [names[i] for i in range(p) if best.ooc_devices >> i & 1],
                "ooc_bytes": best.ooc_bytes,
                "ooc_gb_per_s": best.ooc_bytes / best.t_compute_s / 1e9,
            }
            print(f"n={n:3d} {name}: t={best.t_compute_s:7.3f}s {best.gflops / 1e3:7.1f} TFLOP/s "
                  f"imb={100 * imbalance(per_dev):6.1f}%  "
                  + " ".join(f"{names[i]}={areas[i]}" for i in range(p))
                  + f"  ooc={row[name]['ooc']}", flush=True)
        row["fpm_vs_cpm_time_delta"] = row["fpm"]["t_total_s"] / row["cpm"]["t_total_s"] - 1.0
        row["fpm_vs_homogeneous_time_delta"] = row["fpm"]["t_total_s"] / row["homogeneous"]["t_total_s"] - 1.0
        if "fpm_refined" in row:
            row["fpm_refined_vs_cpm_time_delta"] = row["fpm_refined"]["t_total_s"] / row["cpm"]["t_total_s"] - 1.0
            row["fpm_refined_vs_homogeneous_time_delta"] = (row["fpm_refined"]["t_total_s"] /
                                                             row["homogeneous"]["t_total_s"] - 1.0)
        table.append(row)
    ctx.close()

    out = {
        "config": {"b": b, "ns": ns, "p": p, "names": names, "sm_caps": caps, "cpu_devices": cpu_dev,
                   "c_cap_bytes": c_caps,
                   "ncal": args.ncal, "x_cal": x_cal, "sizes": sizes, "ooc_keep": args.ooc_keep, "ooc_buffers": args.ooc_buffers,
                   "link_group": args.link_group, "refine_rounds": args.refine, "arrange": args.arrange,
                   "cliff_points": args.cliff,
                   "sampling": "concurrent (all devices at once)" if args.concurrent else "exclusive",
                   "dtype": "f32 (auto scheme: F16X3, DESIGN Q15)", "sm_partition": args.sm_partition,
                   "gpu": "1x B200; devices emulated by SM caps, device memory by C caps (C_i out of core above)"},
        "pcie": pcie, "fpm_sample_s": t_sample, "models": sample_info, "table": table,
    }
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps([{"n": r["n"], "fpm_vs_cpm": r["fpm_vs_cpm_time_delta"],
                       "fpm_vs_homogeneous": r["fpm_vs_homogeneous_time_delta"],
                       "fpm_refined_vs_homogeneous": r.get("fpm_refined_vs_homogeneous_time_delta")} for r in table]))


if __name__ == "__main__":
    main()
