#!/usr/bin/env python
"""Hybrid CPU + GPU partition (§VI, Table II P:82-86 and Tables
III / Fig. 7) on one B200 and its host cores.

The paper's node: 4 six-core sockets and 2 GPUs; Table II compares the
multiply on the 24 cores alone (homogeneous distribution), on one GPU with its
dedicated core, and on 22 cores + 2 GPUs partitioned by the FPM-based
algorithm from the speed functions of the GPUs (g1, g2) and of the sockets
(s5, s6).  Here: sockets = CPU devices of c pinned cores each (their host GEMM),
GPU = a GPU device capped to a few SMs so that its speed relative to a socket
is of the paper's order (a whole B200 outruns this host's cores ~200:1), with
a C memory cap so its speed function has the out-of-core cliff of Fig. 3.
One update per pivot (option fuse = 1, the paper's kernel), b = 256.

For each n: "cpus" (the sockets alone, equal areas), "gpu" (the GPU device
alone), and on GPU + sockets: "fpm" (fpm_partition on the sampled speed
functions), "cpm" (constants at the even share of the n_cal problem),
"homogeneous".  Reported: time, GFLOPS, per-device computation time and
areas, FPM vs CPM and homogeneous.  Writes JSON (profiles/hybrid_r02.json).
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

CPU = pkg.FPM_CPU_DEVICE


def imbalance(ts):
    live = [t for t in ts if t > 0]
    return max(live) / (sum(live) / len(live)) - 1.0 if live else 0.0


def timed_run(ctx, N, b, rects, p, reps):
    ctx.setup(N, b, rects, pkg.FPM_F32)
    ctx.fill_synthetic(5, 6, pkg.FPM_DIST_PM1)
    ctx.compute()
    best = None
    for _ in range(reps):
        st = ctx.compute()
        if best is None or st.t_compute_s < best.t_compute_s:
            best = st
    return best, list(best.per_dev_compute_s[:p])


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--b", type=int, default=256)
    ap.add_argument("--ns", default="16,24,32,40,48")
    ap.add_argument("--gpu-sms", type=int, default=2)
    ap.add_argument("--gpu-c-cap-mib", type=int, default=64)
    ap.add_argument("--sockets", default="5,5,5", help="cores per CPU device")
    ap.add_argument("--ncal", type=int, default=16)
    ap.add_argument("--gpu-sizes", default="1,2,4,6,8,10,12,14,16,18,20,24,28,32,36,40,44")
    ap.add_argument("--cpu-sizes", default="1,2,4,8,12,16")
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--refine", type=int, default=0,
                    help="rounds of synchronised level correction (Q26): partition 'fpm_refined'")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "hybrid_r02.json"))
    args = ap.parse_args()
    b = args.b
    sockets = [int(c) for c in args.sockets.split(",")]
    ns = [int(x) for x in args.ns.split(",")]
    gsz = [int(m) ** 2 for m in args.gpu_sizes.split(",")]
    csz = [int(m) ** 2 for m in args.cpu_sizes.split(",")]
    devs = [0] + [CPU] * len(sockets)
    caps = [args.gpu_sms] + sockets
    names = ["G"] + [f"S{i}" for i in range(len(sockets))]
    p = len(devs)
    ctx = pkg.Context.local(devs, sm_caps=caps)
    ctx.set_option("fuse", 1)
    ctx.set_device_option(0, "c_cap_bytes", args.gpu_c_cap_mib << 20)
    t0 = time.perf_counter()
    models = []
    for i in range(p):
        sizes = gsz if i == 0 else csz
        sp = ctx.sample(i, b, sizes, pkg.FPM_F32)[0]
        models.append((sizes, sp))
        print(names[i], " ".join(f"{x}:{s / 1e9:.0f}" for x, s in zip(sizes, sp)), flush=True)
    from studies import refine as rf
    models[0] = rf.cliff_points(ctx, 0, b, models[0], args.gpu_c_cap_mib << 20)   # bracket the GPU's cliff (Q26)
    t_sample = time.perf_counter() - t0
    cpus = pkg.Context.local([CPU] * len(sockets), sm_caps=sockets)
    gpu = pkg.Context.local([0], sm_caps=[args.gpu_sms])
    gpu.set_option("fuse", 1)
    gpu.set_device_option(0, "c_cap_bytes", args.gpu_c_cap_mib << 20)
    for c in (cpus,):
        c.set_option("fuse", 1)
    table = []
    for n in ns:
        N, T = n * b, n * n
        row = {"n": n, "N": N}
        st, per = timed_run(cpus, N, b, pkg.colpart_arrange(n, pkg.fpm_partition(T, [([1], [1.0])] * len(sockets))),
                            len(sockets), args.reps)
        row["cpus"] = {"t_s": st.t_compute_s, "gflops": st.gflops, "imbalance": imbalance(per)}
        st, per = timed_run(gpu, N, b, [(0, 0, 0, n, n)], 1, args.reps)
        row["gpu"] = {"t_s": st.t_compute_s, "gflops": st.gflops, "ooc": bool(st.ooc_devices & 1)}
        x_cal = max(1, args.ncal * args.ncal // p)
        parts = {"fpm": (models, None), "cpm": ([([1], [pkg.fpm_model_speed(m, x_cal)]) for m in models], None),
                 "homogeneous": ([([1], [1.0])] * p, None)}
        if args.refine:
            (x_in, r_in), (x_out, r_out) = rf.cliff_areas(args.gpu_c_cap_mib << 20, b)
            r_models, hist, r_d, r_rects = rf.refine(ctx, n, b, models, args.refine, arrange="fpm", concurrent=True,
                                                      splits=[x_in] + [None] * (p - 1),
                                                      cliffs=[(r_in, r_out)] + [None] * (p - 1))
            parts["fpm_refined"] = (r_models, r_rects)
            row["refine"] = hist
        for name, (mods, given) in parts.items():
            d = pkg.fpm_partition(T, mods)
            rects = given if given is not None else pkg.colpart_arrange(n, d)
            st, per = timed_run(ctx, N, b, rects, p, args.reps)
            row[name] = {"d": d, "areas": [r[3] * r[4] for r in rects], "t_s": st.t_compute_s, "gflops": st.gflops,
                         "per_dev_compute_s": per, "imbalance": imbalance(per), "ooc": bool(st.ooc_devices & 1)}
        row["fpm_vs_cpm"] = row["fpm"]["t_s"] / row["cpm"]["t_s"] - 1
        row["fpm_vs_homogeneous"] = row["fpm"]["t_s"] / row["homogeneous"]["t_s"] - 1
        row["fpm_vs_gpu_alone"] = row["fpm"]["t_s"] / row["gpu"]["t_s"] - 1
        if "fpm_refined" in row:
            row["fpm_refined_vs_cpm"] = row["fpm_refined"]["t_s"] / row["cpm"]["t_s"] - 1
            row["fpm_refined_vs_gpu_alone"] = row["fpm_refined"]["t_s"] / row["gpu"]["t_s"] - 1
        table.append(row)
        ref = row.get("fpm_refined")
        print(f"n={n}: cpus {row['cpus']['t_s']:.3f}s gpu {row['gpu']['t_s']:.3f}s fpm {row['fpm']['t_s']:.3f}s "
              f"(imb {100 * row['fpm']['imbalance']:.1f}%, d={row['fpm']['d']}) "
              + (f"refined {ref['t_s']:.3f}s (imb {100 * ref['imbalance']:.1f}%, d={ref['d']}) " if ref else "")
              + f"cpm {row['cpm']['t_s']:.3f}s homog {row['homogeneous']['t_s']:.3f}s", flush=True)
    for c in (ctx, cpus, gpu):
        c.close()
    out = {"config": {"b": b, "ns": ns, "gpu_sm_cap": args.gpu_sms, "gpu_c_cap_bytes": args.gpu_c_cap_mib << 20,
                      "sockets_cores": sockets, "names": names, "ncal": args.ncal, "fuse": 1,
                      "cpu_isa": pkg.cpu_isa(), "host_cores": len(pkg.cpu_cores()),
                      "dtype": "f32 (GPU F16X3 tcgen05, CPU FP32 FMA)"},
           "fpm_sample_s": t_sample,
           "models": [{"name": nm, "x": m[0], "gflops": [s / 1e9 for s in m[1]]} for nm, m in zip(names, models)],
           "table": table}
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
