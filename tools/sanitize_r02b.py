"""Small invocations of the in-kernel staging paths for
compute-sanitizer (memcheck / racecheck / synccheck): the chunked F16X3 update
whose two staging warps stage the next group (column-maxima atomics, grid
barrier over the staging warps, A rows, B split + transpose), forced on at
sizes the tools finish quickly (option fused_staging = 2), resident
(pmm_compute) and streamed (pmm_run: the staging warps wait for upload-progress
flags), ragged rectangles, several pivots per group, two devices in green
partitions with shared B operands.  SM caps keep every CTA of the persistent
grid resident under instrumentation.  Exits non-zero on a parity failure."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402
import synth  # noqa: E402
from oracle import gemm as og  # noqa: E402


def check(C, A, B, what):
    err = og.rel_fro(C, og.gemm(A, B))
    print(f"{what}: rel_fro={err:.2e}", flush=True)
    assert err <= 1e-5, what


def run(devs, caps, N, b, d, opts, streamed=True):
    n = N // b
    rects = pkg.colpart_arrange(n, d)
    A = synth.rect(1, N, 0, 0, N, N).astype(np.float32)
    B = synth.rect(2, N, 0, 0, N, N).astype(np.float32)
    C = np.full((N, N), np.nan, np.float32)
    with pkg.Context.local(devs, sm_caps=caps) as ctx:
        for k, v in opts.items():
            ctx.set_option(k, v)
        if streamed:
            ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
        else:
            ctx.setup(N, b, rects, pkg.FPM_F32)
            ctx.upload(A, B, N, 0, 0)
            ctx.compute()
            ctx.download(C, N, 0, 0)
    check(C, A, B, f"devs={devs} caps={caps} N={N} b={b} d={d} opts={opts} streamed={streamed}")


FS = {"fused_staging": 2, "e2e_tail": 0}
run([0], [16], 1024, 128, [64], dict(FS, fuse=1), streamed=False)   # 8 groups, resident
run([0], [16], 1024, 128, [64], dict(FS, fuse=1))                    # streamed: progress flags
run([0], [8], 1152, 128, [81], dict(FS, fuse=2))                     # 2 pivots per group, 9 pivots
run([0], [12], 960, 64, [225], dict(FS, fuse=3), streamed=False)      # ragged 960 tiles, odd groups
run([0, 0], [16, 16], 1024, 128, [40, 24], dict(FS, fuse=1, sm_partition=1, share_b=1))  # green, shared B
print("sanitize fused-staging workload ok")
