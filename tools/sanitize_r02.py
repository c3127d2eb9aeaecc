"""Small invocations of the round-2 default paths for compute-sanitizer
(memcheck / racecheck / synccheck): the chunked-accumulation F16X3 update
(variant 8 and 7, overwrite and accumulate, ragged shapes, chunk sizes), TF32X3
on the same kernel, a local multi-device run, a mixed CPU + GPU context, and a
streamed pmm_run.  Exits non-zero on a parity failure."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402
import synth  # noqa: E402
from oracle import gemm as og  # noqa: E402


def run(devs, caps, N, b, d, opts=None, dt=pkg.FPM_F32):
    n = N // b
    rects = pkg.colpart_arrange(n, d)
    npdt = np.float32 if dt == pkg.FPM_F32 else np.float64
    A = synth.rect(1, N, 0, 0, N, N).astype(npdt)
    B = synth.rect(2, N, 0, 0, N, N).astype(npdt)
    C = np.full((N, N), np.nan, npdt)
    with pkg.Context.local(devs, sm_caps=caps) as ctx:
        for k, v in (opts or {}).items():
            ctx.set_option(k, v)
        ctx.run(A, B, C, N, b, rects, dt)
    err = og.rel_fro(C, og.gemm(A, B))
    tol = 1e-5 if dt == pkg.FPM_F32 else 1e-12
    print(f"devs={devs} N={N} b={b} d={d} opts={opts}: rel_fro={err:.2e}", flush=True)
    assert err <= tol


run([0], None, 768, 256, [9])
run([0], None, 800, 160, [25], {"chunk_k": 256})                  # ragged tiles, 2 chunks per fused K
run([0], None, 1024, 256, [16], {"kernel_variant": 7, "e2e_tail": 0})
run([0], None, 512, 128, [16], {"f32_scheme": pkg.SCHEME_TF32X3})
run([0, 0, 0], None, 1024, 128, [40, 14, 10])
run([0, pkg.FPM_CPU_DEVICE], [0, 2], 512, 64, [50, 14])
print("sanitize workload ok")
