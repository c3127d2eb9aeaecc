#!/usr/bin/env python
"""Heterogeneity study (BASELINE config 4 analogue) on ONE B200.

p emulated devices share the GPU, each capped to a number of SMs (the
persistent update kernel's grid), with caps proportional to config 4's
{144, 128, 112, 96, 80, 64, 48, 32} scaled to fit 148 SMs.  For each device an
FPM is sampled with fpm_sample (exclusive, as the paper measures GPUs);
then the same multiply runs under four partitions:

  fpm          fpm_partition on the sampled speed functions ([5])
  cpm_ncal     constant models = speed at the even share of a smaller
               calibration problem N_cal ("when some workload is
               distributed evenly"; P:107 the CPM used speeds measured while the
               problem was small) -- reading Q9
  cpm_self     constant models calibrated at this run's even share
  homogeneous  equal areas

Reported per partition: total time and GFLOPS, per-device computation time
(Fig. 6 metric), measured imbalance max/mean - 1, and the imbalance the
FPMs predict for the achieved areas.  Writes JSON (default profiles/hetero_c4_r01.json).
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


def c4_study(caps, N=32768, b=512, sizes=None, ncal=8192, reps=2, insitu=2, graph=1, sm_partition=0,
             exclusive=True, log=print, refine_rounds=0, options=None, refine_arrange=("paper", "fpm"),
             refine_ci_permille=None) -> dict:
    """Sample each emulated device's FPM, then run the multiply under the FPM,
    CPM (N_cal and self-calibrated), homogeneous and in-situ corrected FPM
    partitions; returns the result dict written by main()."""
    p = len(caps)
    n = N // b
    T = n * n
    sizes = sizes or [m * m for m in (1, 2, 3, 4, 6, 8, 12, 16, 20, 24, 28, 32, 40)]

    ctx = pkg.Context.local([0] * p, sm_caps=caps)
    ctx.set_option("sm_partition", sm_partition)
    ctx.set_option("graph", graph)
    for k, v in (options or {}).items():
        ctx.set_option(k, v)
    t0 = time.perf_counter()
    models, sample_info = [], []
    if exclusive:   # each device alone (how the paper measured its GPUs)
        per_dev = [ctx.sample(dev, b, sizes, pkg.FPM_F32) for dev in range(p)]
    else:           # all devices at once (P:10 (ii)): contention as in the run
        sps, cis, repss = ctx.sample(-1, b, sizes, pkg.FPM_F32)
        per_dev = list(zip(sps, cis, repss))
    for dev, (sp, ci, nrep) in enumerate(per_dev):
        models.append((sizes, sp))
        sample_info.append({"cap": caps[dev], "speeds_gflops": [s / 1e9 for s in sp], "rel_ci95": ci, "reps": nrep})
    t_sample = time.perf_counter() - t0

    x_cal = max(1, (ncal // b) ** 2 // p)
    x_even = T // p
    parts = {
        "fpm": pkg.fpm_partition(T, models),
        "cpm_ncal": pkg.fpm_partition(T, [([1], [pkg.fpm_model_speed(m, x_cal)]) for m in models]),
        "cpm_self": pkg.fpm_partition(T, [([1], [pkg.fpm_model_speed(m, x_even)]) for m in models]),
        "homogeneous": pkg.fpm_partition(T, [([1], [1.0])] * p),
    }
    results = {}

    def corrected(mods, res):
        """Each device's model scaled by (speed it achieved in the run at its
        area) / (model speed there): the models keep their shape (P:8), their
        levels absorb the contention of the concurrent run.  The partition is
        invariant to a common factor, so only the relative corrections act."""
        out = []
        for m, a, t in zip(mods, res["areas"], res["per_dev_compute_s"]):
            if a <= 0 or t <= 0:
                out.append(m)
                continue
            r = (2.0 * a * b * b * N / t) / pkg.fpm_model_speed(m, a)
            out.append((m[0], [s * r for s in m[1]]))
        return out

    # operating-point refinement (reading Q26): every device timed on its own
    # rectangle, all at once, points added to the models, partition repeated
    refined = {}
    if refine_rounds > 0:
        from studies import refine as rf
        for arr in refine_arrange:
            mods_r, hist, d_r, rects_r = rf.refine(ctx, n, b, models, refine_rounds, arrange=arr, log=log,
                                                   ci_permille=refine_ci_permille)
            # (synchronised level correction of the exclusive models, Q26)
            refined["fpm_refined" + ("_arr" if arr == "fpm" else "")] = (mods_r, hist, d_r, rects_r)

    # "_arr": the same partition arranged by colpart_arrange_fpm (integer widths
    # and heights chosen on the models, reading Q25) instead of colpart_arrange
    order = [("fpm", parts["fpm"]), ("fpm_arr", parts["fpm"])]
    order += [(k, v[2]) for k, v in refined.items()]
    order += [(k, v) for k, v in parts.items() if k != "fpm"]
    for it in range(insitu):
        order += [(f"fpm_insitu{it + 1}", None), (f"fpm_insitu{it + 1}_arr", None)]
    cur_models = models
    for name, d in order:
        if d is None and not name.endswith("_arr"):   # in-situ corrected FPMs from the previous FPM run
            prev = results["fpm" if name == "fpm_insitu1" else f"fpm_insitu{int(name[-1]) - 1}"]
            cur_models = corrected(cur_models, prev)
        if d is None:
            d = pkg.fpm_partition(T, cur_models)
        if name in refined:
            rects = refined[name][3]
        elif name.endswith("_arr"):
            rects = pkg.colpart_arrange_fpm(n, d, cur_models if name.startswith("fpm_insitu") else models)
        else:
            rects = pkg.colpart_arrange(n, d)
        ctx.setup(N, b, rects, pkg.FPM_F32)
        ctx.fill_synthetic(5, 6, pkg.FPM_DIST_PM1)
        ctx.compute()
        best = None
        for _ in range(reps):
            st = ctx.compute()
            if best is None or st.t_compute_s < best.t_compute_s:
                best = st
        areas = [r[3] * r[4] for r in rects]
        per_dev = list(best.per_dev_compute_s[:p])
        spans = list(best.per_dev_span_s[:p])
        # FPM-predicted k-loop time: 2 a b^2 N flop at the model's speed s(a)
        pred_models = (refined[name][0] if name in refined else
                       cur_models if name.startswith("fpm_insitu") else models)
        pred = [2.0 * a * b * b * N / pkg.fpm_model_speed(m, a) if a > 0 else 0.0
                for a, m in zip(areas, pred_models)]
        results[name] = {
            "d": d, "areas": areas, "rects": rects,
            "t_total_s": best.t_compute_s, "gflops": best.gflops,
            "per_dev_compute_s": per_dev,
            "imbalance_measured": imbalance(per_dev), "imbalance_predicted": imbalance(pred),
            "per_dev_span_s": spans, "imbalance_span": imbalance([t for t, a in zip(spans, areas) if a > 0]),
            "per_dev_update_s": list(best.per_dev_update_s[:p]),
            "predicted_time_s": max(pred),
            "comm_bytes": best.comm_bytes,
        }
        if name in refined:
            results[name]["refine_history"] = refined[name][1]
        log(f"{name:12s} t={best.t_compute_s:8.4f}s  {best.gflops / 1e3:8.1f} TFLOP/s  "
            f"imb meas={100 * imbalance(per_dev):6.2f}%  pred={100 * imbalance(pred):6.2f}%  d={d}")
    ctx.close()

    # reference: the whole GPU as one device (upper bound of the aggregate)
    with pkg.Context.local([0]) as one:
        one.setup(N, b, [(0, 0, 0, n, n)], pkg.FPM_F32)
        one.fill_synthetic(5, 6, pkg.FPM_DIST_PM1)
        one.compute()
        st1 = one.compute()
    return {
        "config": {"N": N, "b": b, "p": p, "sm_caps": list(caps), "ncal": ncal, "x_cal": x_cal, "x_even": x_even,
                   "sizes": sizes, "dtype": "f32 (auto scheme: F16X3, DESIGN Q15)", "sm_partition": sm_partition,
                   "gpu": "1x B200, devices emulated by SM caps",
                   "sampling": "exclusive" if exclusive else "concurrent (all devices at once)"},
        "fpm_sample_s": t_sample, "models": sample_info, "partitions": results,
        "whole_gpu": {"t_s": st1.t_compute_s, "gflops": st1.gflops},
        "fpm_vs_cpm_ncal_time_delta": results["fpm"]["t_total_s"] / results["cpm_ncal"]["t_total_s"] - 1.0,
        "fpm_vs_homogeneous_time_delta": results["fpm"]["t_total_s"] / results["homogeneous"]["t_total_s"] - 1.0,
    }


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--N", type=int, default=32768)
    ap.add_argument("--b", type=int, default=512)
    ap.add_argument("--caps", default="30,26,24,20,16,14,10,6")
    ap.add_argument("--ncal", type=int, default=8192)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--sizes", default="1,2,3,4,6,8,12,16,20,24,28,32,40")
    ap.add_argument("--concurrent", dest="exclusive", action="store_false",
                    help="sample all devices at once (P:10 (ii)) instead of each alone (P:11, default)")
    ap.add_argument("--insitu", type=int, default=2,
                    help="extra FPM partitions with models rescaled by the speeds achieved in the previous run")
    ap.add_argument("--graph", type=int, default=1, help="pmm_compute as a replayed CUDA graph (option graph)")
    ap.add_argument("--sm-partition", type=int, default=0,
                    help="1 = each device in its own green-context SM partition (all its kernels confined)")
    ap.add_argument("--refine", type=int, default=0, help="rounds of operating-point refinement (Q26)")
    ap.add_argument("--option", action="append", default=[], help="context option key=value (repeatable)")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "hetero_c4_r01.json"))
    args = ap.parse_args()
    caps = [int(c) for c in args.caps.split(",")]
    out = c4_study(caps, args.N, args.b, [int(m) ** 2 for m in args.sizes.split(",")], args.ncal, args.reps,
                   args.insitu, args.graph, args.sm_partition, args.exclusive, log=lambda s: print(s, flush=True),
                   refine_rounds=args.refine,
                   options={kv.split("=")[0]: int(kv.split("=")[1]) for kv in args.option})
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps({k: out[k] for k in ("fpm_vs_cpm_ncal_time_delta", "fpm_vs_homogeneous_time_delta")}))


if __name__ == "__main__":
    main()
