#!/usr/bin/env python
"""Resource contention between a GPU and the host cores of its node (PAPER.md
§III P:11 and Fig. 5, P:68 / P:77-78).

The paper measured (i) the speed of 5 cores of a socket executing the GEMM
kernel while the GPU on the same socket executed its kernel, against the same
cores alone, and (ii) the GPU's speed while the cores were busy, against the
GPU alone: "the performance of the GPU dropped by 7-15% because of resource
contention, while the CPU cores were not so much affected", and the
GPU's exclusive FPM approximated its contended speed "with 85% accuracy".

Here: a CPU device of c pinned cores (cores 1.., core 0 drives the GPU as in
P:11) runs its host GEMM (fpm_k_cpu_gemm's kernel) and a GPU device runs the
tcgen05 update, each sampled with fpm_sample (the paper's statistically
reliable repetition, Q8) alone and then while the other device runs its
kernel continuously in a background thread (the library calls release the
GIL).  Two GPU set-ups: C_i resident in HBM (the B200 default: the GPU's kernel
touches no host resource) and C_i out of core (pmm_set_device_option
"c_cap_bytes": C streamed over PCIe through host memory every update, the
paper's kernel versions 2/3) -- the set-up in which the paper saw the
contention.  Writes JSON (default profiles/contention_r02.json).
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import threading
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

CPU = pkg.FPM_CPU_DEVICE


class Background:
    """Runs `fn` in a loop on a thread until stopped (the other device's load)."""

    def __init__(self, fn):
        self.fn, self.stop_flag, self.calls = fn, False, 0
        self.t = threading.Thread(target=self._loop, daemon=True)

    def _loop(self):
        while not self.stop_flag:
            self.fn()
            self.calls += 1

    def __enter__(self):
        self.t.start()
        time.sleep(0.5)   # the load is running before the measurement starts
        return self

    def __exit__(self, *exc):
        self.stop_flag = True
        self.t.join()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--b", type=int, default=512)
    ap.add_argument("--cores", type=int, default=0, help="CPU device cores (0: all but the GPU's core)")
    ap.add_argument("--gpu-sms", type=int, default=0, help="SM cap of the GPU device (0: all)")
    ap.add_argument("--gpu-sizes", default="4,8,16,24,32,40")
    ap.add_argument("--cpu-sizes", default="1,2,3,4,6")
    ap.add_argument("--ooc-cap-mib", type=int, default=256, help="C cap of the out-of-core GPU set-up")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "contention_r02.json"))
    args = ap.parse_args()
    b = args.b
    ncores = len(pkg.cpu_cores())
    cores = args.cores or (ncores - 1)
    gpu_sizes = [int(m) ** 2 for m in args.gpu_sizes.split(",")]
    cpu_sizes = [int(m) ** 2 for m in args.cpu_sizes.split(",")]
    out = {"config": {"b": b, "cpu_cores": cores, "host_cores": ncores, "cpu_isa": pkg.cpu_isa(),
                      "gpu_sm_cap": args.gpu_sms, "gpu_sizes": gpu_sizes, "cpu_sizes": cpu_sizes,
                      "dtype": "f32 (GPU: F16X3 tcgen05; CPU: FP32 FMA GEMM)",
                      "ooc_cap_bytes": args.ooc_cap_mib << 20}, "setups": {}}

    with pkg.Context.local([CPU], sm_caps=[cores]) as cctx:
        # the socket's load while the GPU is measured: its kernel at a mid size, continuously
        cpu_load = lambda: cctx.sample(0, b, [cpu_sizes[len(cpu_sizes) // 2]], pkg.FPM_F32)  # noqa: E731
        cpu_alone = cctx.sample(0, b, cpu_sizes, pkg.FPM_F32)[0]
        print("cpu alone  ", [round(s / 1e9, 1) for s in cpu_alone], flush=True)
        for setup, cap in (("gpu_resident", 0), ("gpu_out_of_core", args.ooc_cap_mib << 20)):
            with pkg.Context.local([0], sm_caps=[args.gpu_sms]) as gctx:
                if cap:
                    gctx.set_device_option(0, "c_cap_bytes", cap)
                gpu_load = lambda: gctx.sample(0, b, [gpu_sizes[-1]], pkg.FPM_F32)  # noqa: E731
                g_alone = gctx.sample(0, b, gpu_sizes, pkg.FPM_F32)[0]
                with Background(cpu_load) as bg:
                    g_loaded = gctx.sample(0, b, gpu_sizes, pkg.FPM_F32)[0]
                g_bg_calls = bg.calls
                with Background(gpu_load) as bg:
                    c_loaded = cctx.sample(0, b, cpu_sizes, pkg.FPM_F32)[0]
                c_bg_calls = bg.calls
            rec = {
                "gpu_alone_gflops": [s / 1e9 for s in g_alone],
                "gpu_with_cpu_load_gflops": [s / 1e9 for s in g_loaded],
                "gpu_drop_pct": [100.0 * (1 - l / a) for a, l in zip(g_alone, g_loaded)],
                "cpu_alone_gflops": [s / 1e9 for s in cpu_alone],
                "cpu_with_gpu_load_gflops": [s / 1e9 for s in c_loaded],
                "cpu_drop_pct": [100.0 * (1 - l / a) for a, l in zip(cpu_alone, c_loaded)],
                "background_calls": {"cpu_load_during_gpu": g_bg_calls, "gpu_load_during_cpu": c_bg_calls},
            }
            out["setups"][setup] = rec
            print(setup, "gpu drop %", [round(v, 1) for v in rec["gpu_drop_pct"]],
                  "cpu drop %", [round(v, 1) for v in rec["cpu_drop_pct"]], flush=True)
    os.makedirs(os.path.dirname(args.out), exist_ok=True)
    with open(args.out, "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
