#!/usr/bin/env python
"""Config 2 (BASELINE.json): single-B200 speed functions of the rank-b update.

(1) Standalone kernel curve (the Fig. 3 analogue): the update kernel
    alone, C_i += A(b) B(b) with an L x L C and K = b in {512, 64}, L from 64 to
    16384 (x1.5 / x2 steps), uncapped and SM-capped; GFLOPS and fraction of the
    tensor roofline of the FP32 scheme (--scheme: f16x3 default, f16i8).  Timed with CUDA events on the launching stream over
    repeated launches (inputs resident; C is 1 GB at L = 16384).
(2) Model points: fpm_sample at x = m^2 blocks (m = 1..32, b = 512), i.e. the
    FPM the partitioner consumes (P:18 sqrt(x) x sqrt(x)).

Writes profiles/speed_sweep_r02_<scheme>.json.
"""
from __future__ import annotations

import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

L_LIST = [64, 96, 128, 192, 256, 384, 512, 768, 1024, 1536, 2048, 3072, 4096, 6144, 8192, 12288, 16384]


SCHEMES = {"f16i8": (3, 2.0, "measured bf16 dense / 2 (F16I8: one fp16 MMA + one int8 MMA of 2K at 2x rate)"),
           "f16x3": (0, 3.0, "measured bf16 dense / 3 (F16X3: three fp16 MMAs per FP32 MAC)")}


def peak_alg_tflops(per_mac):
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    d = json.load(open(path)) if os.path.exists(path) else {}
    return d.get("bf16_tflops", 1590.0) / per_mac, d.get("bf16_tflops_sustained", 1400.0) / per_mac


def time_update(L, K, cap, scheme, reps=20):
    dev = torch.device("cuda")
    A = torch.empty((L, K), device=dev)
    B = torch.empty((K, L), device=dev)
    pkg.k_fill_synthetic(A, pkg.FPM_F32, K, 1, 1 << 20, 0, 0, L, K)
    pkg.k_fill_synthetic(B, pkg.FPM_F32, L, 2, 1 << 20, 0, 0, K, L)
    ah = torch.empty((L, K), dtype=torch.float16, device=dev)
    al = torch.empty_like(ah)
    bh = torch.empty((L, K), dtype=torch.float16, device=dev)
    bl = torch.empty_like(bh)
    sa = torch.empty(L, device=dev)
    sb = torch.empty(L, device=dev)
    pkg.k_split_f32(A, K, L, K, scheme, ah, al, sa)
    pkg.k_split_cols_f32(B, L, K, L, scheme, bh, bl, sb)
    C = torch.zeros((L, L), device=dev)
    for _ in range(3):
        pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, L, L, K, L, scheme=scheme, num_sms=cap)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(reps):
        pkg.k_update_f32(ah, al, bh, bl, sa, sb, C, L, L, K, L, scheme=scheme, num_sms=cap)
    e1.record()
    torch.cuda.synchronize()
    t = e0.elapsed_time(e1) * 1e-3 / reps
    return 2.0 * L * L * K / t


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--caps", default="0,74,30")
    ap.add_argument("--scheme", choices=sorted(SCHEMES), default="f16x3")
    ap.add_argument("--out", default=None)
    args = ap.parse_args()
    scheme, per_mac, basis = SCHEMES[args.scheme]
    if args.out is None:
        args.out = os.path.join(ROOT, "profiles", f"speed_sweep_r02_{args.scheme}.json")
    caps = [int(c) for c in args.caps.split(",")]
    burst, sustained = peak_alg_tflops(per_mac)
    torch.cuda.set_device(0)
    curves = []
    for cap in caps:
        for K in (512, 64):
            pts = []
            for L in L_LIST:
                g = time_update(L, K, cap, scheme)
                scale = (cap if cap else 148) / 148.0
                pts.append({"L": L, "gflops": g / 1e9, "frac_burst_peak": g / 1e12 / (burst * scale)})
                print(f"cap={cap or 148:3d} K={K:4d} L={L:6d} {g / 1e12:8.2f} TFLOP/s "
                      f"({100 * g / 1e12 / (burst * scale):5.1f}% of capped burst peak)", flush=True)
            curves.append({"sm_cap": cap or 148, "K": K, "points": pts})
    models = []
    with pkg.Context.local([0] * len(caps), sm_caps=[c for c in caps]) as ctx:
        ctx.set_option("f32_scheme", scheme)
        sizes = [m * m for m in range(1, 33)]
        for dev, cap in enumerate(caps):
            sp, ci, reps = ctx.sample(dev, 512, sizes, pkg.FPM_F32)
            models.append({"sm_cap": cap or 148, "b": 512, "x": sizes, "speed_gflops": [s / 1e9 for s in sp],
                           "rel_ci95": ci, "reps": reps})
    out = {"peak_alg_tflops": {"burst": burst, "sustained": sustained,
                               "basis": basis}, "scheme": args.scheme,
           "kernel_curves": curves, "fpm_models": models}
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    json.dump(out, open(args.out, "w"), indent=1)


if __name__ == "__main__":
    main()
