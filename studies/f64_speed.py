#!/usr/bin/env python
"""FP64 rank-b update (config 1 precision) throughput on one B200: the DMMA
kernel alone, C (L x L) += A (L x K) Bt^T, for a few L and K.  Reported against
the B200 FP64 tensor peak (nominal ~40 TFLOP/s; no measured FP64 peak exists in
MEASURED_PEAKS.json)."""
from __future__ import annotations

import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

NOMINAL_FP64_TFLOPS = 40.0


def cublas_dgemm_tflops(n: int = 8192) -> float:
    """Library reference for the FP64 denominator: torch.matmul (cuBLAS DGEMM)."""
    a = torch.randn((n, n), dtype=torch.float64, device="cuda")
    b = torch.randn((n, n), dtype=torch.float64, device="cuda")
    for _ in range(2):
        torch.matmul(a, b)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(5):
        torch.matmul(a, b)
    e1.record()
    torch.cuda.synchronize()
    return 2.0 * n ** 3 / (e0.elapsed_time(e1) * 1e-3 / 5) / 1e12


def main():
    torch.cuda.set_device(0)
    ref = cublas_dgemm_tflops()
    print(f"cuBLAS DGEMM 8192^3: {ref:.2f} TFLOP/s", flush=True)
    out = [{"cublas_dgemm_8192_tflops": ref}]
    for K in (64, 512):
        for L in (512, 1024, 2048, 4096, 8192):
            A = torch.empty((L, K), dtype=torch.float64, device="cuda")
            Bt = torch.empty((L, K), dtype=torch.float64, device="cuda")
            pkg.k_fill_synthetic(A, pkg.FPM_F64, K, 1, 1 << 20, 0, 0, L, K)
            pkg.k_fill_synthetic(Bt, pkg.FPM_F64, K, 2, 1 << 20, 0, 0, L, K)
            C = torch.zeros((L, L), dtype=torch.float64, device="cuda")
            for _ in range(3):
                pkg.k_update_f64(A, K, Bt, C, L, L, K, L)
            reps = 10
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            torch.cuda.synchronize()
            e0.record()
            for _ in range(reps):
                pkg.k_update_f64(A, K, Bt, C, L, L, K, L)
            e1.record()
            torch.cuda.synchronize()
            t = e0.elapsed_time(e1) * 1e-3 / reps
            tf = 2.0 * L * L * K / t / 1e12
            out.append({"L": L, "K": K, "tflops": tf, "frac_nominal": tf / NOMINAL_FP64_TFLOPS,
                        "frac_cublas": tf / ref})
            print(f"K={K:4d} L={L:5d} {tf:7.2f} TFLOP/s  ({100 * tf / NOMINAL_FP64_TFLOPS:5.1f}% of nominal 40, "
                  f"{100 * tf / ref:5.1f}% of cuBLAS DGEMM)", flush=True)
    if len(sys.argv) > 1:
        json.dump(out, open(sys.argv[1], "w"), indent=1)


if __name__ == "__main__":
    main()
