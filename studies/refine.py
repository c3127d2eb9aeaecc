"""Operating-point refinement of the FPMs (reading Q26).

The speed functions are sampled in advance on sqrt(x) x sqrt(x) submatrices
(P:18).  Between two sample sizes the model is a straight segment, which
misses a memory cliff that lies between them, and each device was timed alone,
so resources shared in the run (a host link, the power budget of a GPU that
several emulated devices share) are not in the model.  Refinement: partition,
arrange, then time every device on the very rectangle it was given -- all
devices at once (P:10 (ii): "processes are synchronised ... the resources will
be shared between the maximum number of processes") -- add those points to the
models (the speed does not vary with the nearly square shapes, so a
rectangle of area h w is a sample of x = h w) and repeat until the partition
stops changing.  This is the partial-model idea of [5]: the model is
made exact where the partitioner looks.

Orchestration only: sampling (fpm_sample_rects), partitioning and arranging
are library calls.
"""
from __future__ import annotations

import paper_conf_cluster_zhongrl12_b200 as pkg


def add_point(model, x, s):
    """Model (xs, ss) with the point (x, s) inserted (or replacing x)."""
    xs, ss = list(model[0]), list(model[1])
    if x in xs:
        ss[xs.index(x)] = s
    else:
        k = sum(1 for v in xs if v < x)
        xs.insert(k, x)
        ss.insert(k, s)
    return xs, ss


def refine(ctx, n, b, models, rounds=3, arrange="paper", concurrent=True, dtype=pkg.FPM_F32, log=None):
    """Returns (refined models, history, d, rects) for T = n^2 blocks.
    arrange: "paper" (colpart_arrange) or "fpm" (colpart_arrange_fpm on the
    current models).  concurrent: sample all devices at once (fpm_sample_rects
    dev = -1; contexts with CPU devices sample each device alone)."""
    T = n * n
    p = len(models)
    mods = [(list(xs), list(ss)) for xs, ss in models]

    def place(m):
        d = pkg.fpm_partition(T, m)
        r = pkg.colpart_arrange_fpm(n, d, m) if arrange == "fpm" else pkg.colpart_arrange(n, d)
        return d, r

    d, rects = place(mods)
    hist = []
    for it in range(rounds):
        shapes = [[(max(1, r[3]), max(1, r[4]))] for r in rects]
        if concurrent:
            sp, _, _ = ctx.sample_rects(-1, b, shapes, dtype)
            sp = [row[0] for row in sp]
        else:
            sp = [ctx.sample_rects(i, b, shapes[i], dtype)[0][0] for i in range(p)]
        for i, r in enumerate(rects):
            if r[3] * r[4] > 0:
                mods[i] = add_point(mods[i], r[3] * r[4], sp[i])
        hist.append({"round": it, "d": list(d), "areas": [r[3] * r[4] for r in rects],
                     "sampled_gflops": [v / 1e9 for v in sp]})
        d_new, rects_new = place(mods)
        if log:
            log(f"refine {it}: d={d} -> {d_new}")
        if d_new == d:
            break
        d, rects = d_new, rects_new
    return mods, hist, d, rects
