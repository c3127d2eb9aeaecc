#!/usr/bin/env python
"""BASELINE.json configs on ONE B200 (what one GPU can run; multi-GPU configs
with devices emulated by SM caps — each device a persistent update grid of
`cap` SMs — run concurrently on the same GPU):

  c1  N = 512, b = 64, FP64, 2 devices in disjoint green partitions {100, 48}: FPMs from 8 sample
      sizes -> fpm_partition -> colpart_arrange -> pmm_run (host A, B, C),
      checked against the CPU oracle (rel-Fro <= 1e-12), oracle time reported.
  c3  N = 16384, b = 512, FP32: p = 1 on the whole GPU; p = 2, 4, 8 homogeneous
      emulated devices (148 / p SMs each) -- exercises the column arrangement
      and the pivot exchange at this size.
  c5  N = 49152, b = 1024, FP32, p = 1.

(c2 = studies/speed_sweep.py, c4 = studies/hetero.py.)  Sampled parity at
full size: blocks of C against the oracle.  Writes profiles/configs_r01.json.
"""
from __future__ import annotations

import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402
import synth  # noqa: E402
from oracle import gemm as og  # noqa: E402


def sampled_parity(ctx, N, seeds, rects, b, nblocks=4):
    rng = np.random.default_rng(N)
    worst = 0.0
    for i, r in enumerate(rects):
        if r[3] * r[4] == 0:
            continue
        R0, C0, H, W = r[1] * b, r[2] * b, r[3] * b, r[4] * b
        for _ in range(nblocks // 2 or 1):
            r0 = R0 + int(rng.integers(0, max(1, H - 8)))
            c0 = C0 + int(rng.integers(0, max(1, W - 32)))
            h, w = min(8, R0 + H - r0), min(32, C0 + W - c0)
            got = ctx.download_block(r0, c0, h, w)
            ref = og.gemm(synth.rect(seeds[0], N, r0, 0, h, N), synth.rect(seeds[1], N, 0, c0, N, w))
            worst = max(worst, og.rel_fro(got, ref))
    return worst


def c1():
    N, b = 512, 64
    n = N // b
    sizes = [m * m for m in range(1, 9)]
    sa, sb = synth.seeds_for_config(0)
    A = synth.rect(sa, N, 0, 0, N, N, dtype=np.float64)
    B = synth.rect(sb, N, 0, 0, N, N, dtype=np.float64)
    with pkg.Context.local([0, 0], sm_caps=[100, 48]) as ctx:
        ctx.set_option("sm_partition", 1)   # disjoint SM partitions (reading Q13)
        models = [(sizes, ctx.sample(dev, b, sizes, pkg.FPM_F64)[0]) for dev in range(2)]
        t0 = time.perf_counter()
        d = pkg.fpm_partition(n * n, models)
        rects = pkg.colpart_arrange(n, d)
        t_host = time.perf_counter() - t0
        C = np.zeros((N, N))
        ctx.run(A, B, C, N, b, rects, pkg.FPM_F64)  # warm-up
        t0 = time.perf_counter()
        st = ctx.run(A, B, C, N, b, rects, pkg.FPM_F64)
        t_run = time.perf_counter() - t0
    t0 = time.perf_counter()
    ref = og.gemm(A, B)
    t_oracle = time.perf_counter() - t0
    return {"N": N, "b": b, "dtype": "f64", "sm_caps": [100, 48], "sm_partition": 1, "partition": d, "rects": rects,
            "models_gflops": [[s / 1e9 for s in m[1]] for m in models],
            "host_partition_arrange_s": t_host, "pmm_run_wall_s": t_run, "k_loop_s": st.t_compute_s,
            "rel_fro": og.rel_fro(C, ref), "oracle_s": t_oracle, "oracle_threads": og.num_threads()}


def run_device_resident(N, b, caps, reps=3, arrange="paper"):
    p = len(caps)
    n = N // b
    sa, sb = synth.seeds_for_config(2 if N == 16384 else 4)
    models = [([1], [float(c or 148)]) for c in caps]
    d = pkg.fpm_partition(n * n, models)
    # paper: colpart_arrange (rounded quotas); fpm: colpart_arrange_fpm (reading Q25)
    rects = pkg.colpart_arrange(n, d) if arrange == "paper" else pkg.colpart_arrange_fpm(n, d, models)
    with pkg.Context.local([0] * p, sm_caps=caps if p > 1 else None) as ctx:
        ctx.setup(N, b, rects, pkg.FPM_F32)
        ctx.fill_synthetic(sa, sb)
        ctx.compute()
        best = None
        for _ in range(reps):
            st = ctx.compute()
            if best is None or st.t_compute_s < best.t_compute_s:
                best = st
        err = sampled_parity(ctx, N, (sa, sb), rects, b)
    per = list(best.per_dev_compute_s[:p])
    live = [t for t in per if t > 0]
    return {"N": N, "b": b, "p": p, "sm_caps": caps, "arrange": arrange, "partition": d, "rects": rects,
            "t_s": best.t_compute_s, "tflops": best.gflops / 1e3, "updates": best.updates,
            "imbalance": max(live) / (sum(live) / len(live)) - 1.0, "comm_bytes": best.comm_bytes,
            "sampled_rel_fro_max": err}


def main():
    out = {"c1": c1()}
    print("c1", {k: out["c1"][k] for k in ("partition", "rel_fro", "pmm_run_wall_s", "oracle_s")}, flush=True)
    out["c3"] = []
    for p, arrange in ((1, "paper"), (2, "paper"), (4, "paper"), (8, "paper"), (8, "fpm")):
        caps = [0] if p == 1 else [148 // p // 2 * 2] * p
        r = run_device_resident(16384, 512, caps, arrange=arrange)
        out["c3"].append(r)
        print("c3", p, arrange, round(r["tflops"], 1), "TFLOP/s", "imb %.2f%%" % (100 * r["imbalance"]),
              "err %.1e" % r["sampled_rel_fro_max"], [x[3] * x[4] for x in r["rects"]], flush=True)
    r = run_device_resident(49152, 1024, [0])
    out["c5"] = r
    print("c5", round(r["tflops"], 1), "TFLOP/s", "err %.1e" % r["sampled_rel_fro_max"], flush=True)
    path = sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "profiles", "configs_r01.json")
    json.dump(out, open(path, "w"), indent=1)


if __name__ == "__main__":
    main()
