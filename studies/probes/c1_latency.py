"""Config 1 (N = 512, b = 64, FP64, 2 devices capped {144, 48}): k-loop time of
pmm_run (eager, host-streamed) and of pmm_compute (resident, CUDA graph), for
fuse = 1 (one rank-b update per pivot) and auto (8 pivots per update)."""
import os
import sys

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), "..", ".."))
import numpy as np  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402
import synth  # noqa: E402
from oracle import gemm as og  # noqa: E402

N, b = 512, 64
n = N // b
A = synth.rect(1, N, 0, 0, N, N, dtype=np.float64)
B = synth.rect(2, N, 0, 0, N, N, dtype=np.float64)
ref = og.gemm(A, B)
rects = pkg.colpart_arrange(n, [32, 32])
for fuse in (1, 0):
    with pkg.Context.local([0, 0], sm_caps=[144, 48]) as ctx:
        ctx.set_option("fuse", fuse)
        C = np.zeros((N, N))
        for _ in range(3):
            st = ctx.run(A, B, C, N, b, rects, pkg.FPM_F64)
        err = og.rel_fro(C, ref)
        ctx.upload(A, B, N)
        ts = sorted(ctx.compute().t_compute_s for _ in range(10))
        print(f"fuse={fuse or 'auto'}: pmm_run k-loop {st.t_compute_s * 1e6:.0f} us ({st.updates} updates), "
              f"pmm_compute (graph) median {ts[5] * 1e6:.0f} us, rel_fro {err:.1e}", flush=True)
