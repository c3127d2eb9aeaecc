"""FPM construction helpers beyond the square size sweep (reading Q26).

The speed functions are sampled in advance on sqrt(x) x sqrt(x) submatrices
(P:18), each device alone.  Two things such a model can miss:

1. **A memory cliff between two sample sizes.**  A device whose C_i must fit a
   memory cap is fast up to x_in = cap / (b^2 s) blocks and out of core above
   (Fig. 3).  With squares only, the cliff lies between m^2 and
   (m+1)^2 and the linear segment across it promises intermediate speeds that
   do not exist.  `cliff_points` samples the largest in-core area and the
   smallest out-of-core area as nearly square rectangles (the speed "does
   not vary with the nearly square shapes") and adds them, so the model drops
   within a few blocks, where the device does.

2. **Resources shared in the run.**  Devices measured alone do not see the
   host link, power budget or memory system they share with the others when
   all run (P:10 (ii): measure "synchronised" processes, so "the resources
   will be shared between the maximum number of processes").  `refine` times
   every device on the very rectangle the partition gave it, all devices at
   once (fpm_sample_rects dev = -1: each repeats its kernel to fill a common
   window), and rescales the device's model by measured / modelled speed at
   that point -- the shape stays the one of the size sweep, the level becomes
   the synchronised one; for a capped device only the points on the same side
   of its cliff -- then re-partitions, until the partition stops changing; if it
   does not within the rounds, the candidate with the smallest measured
   makespan is kept.

Orchestration only: sampling (fpm_sample / fpm_sample_rects), partitioning and
arranging are library calls.
"""
from __future__ import annotations

import math

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


def near_square(x, max_aspect=2.0):
    """A rectangle (h, w), h <= w, h w = x, with the smallest aspect ratio
    w / h <= max_aspect, or None."""
    best = None
    for h in range(int(math.isqrt(x)), 0, -1):
        if x % h == 0:
            w = x // h
            if w / h <= max_aspect:
                best = (h, w)
            break
    return best


def cliff_areas(cap_bytes, b, es=4, max_aspect=2.0):
    """(largest in-core area, smallest out-of-core area) in blocks, each with a
    nearly square rectangle: ((x_in, (h, w)), (x_out, (h, w)))."""
    x_cap = cap_bytes // (b * b * es)
    x_in = x_cap
    while x_in > 0 and near_square(x_in, max_aspect) is None:
        x_in -= 1
    x_out = x_cap + 1
    while near_square(x_out, max_aspect) is None:
        x_out += 1
    return (x_in, near_square(x_in, max_aspect)), (x_out, near_square(x_out, max_aspect))


def cliff_points(ctx, dev, b, model, cap_bytes, dtype=pkg.FPM_F32, es=4):
    """Model with the two points that bracket device dev's memory cliff."""
    (x_in, r_in), (x_out, r_out) = cliff_areas(cap_bytes, b, es)
    shapes = [r for r in (r_in, r_out) if r is not None]
    sp, _, _ = ctx.sample_rects(dev, b, shapes, dtype)
    m = model
    for (x, _), s in zip([p for p in ((x_in, r_in), (x_out, r_out)) if p[1] is not None], sp):
        m = add_point(m, x, s)
    return m


def rescale(model, x_op, s_op, split=None):
    """The model times s_op / model(x_op): all points, or -- with a cliff at
    `split` (largest in-core area) -- those on x_op's side of it."""
    r = s_op / pkg.fpm_model_speed(model, x_op)
    xs, ss = list(model[0]), list(model[1])
    for i, x in enumerate(xs):
        if split is None or (x <= split) == (x_op <= split):
            ss[i] *= r
    return xs, ss, r


def refine(ctx, n, b, models, rounds=3, arrange="paper", concurrent=True, dtype=pkg.FPM_F32, splits=None,
           cliffs=None, log=None, ci_permille=None):
    """Synchronised level correction: returns (models, history, d, rects) for
    T = n^2 blocks.  arrange: "paper" (colpart_arrange) or "fpm"
    (colpart_arrange_fpm on the current models); concurrent: sample all devices
    at once (with CPU devices: every device on its own host thread, windows in
    step); splits: per device
    the largest in-core area (None: no cliff); cliffs: per device the two
    bracketing rectangles ((h, w) in core, (h, w) out of core) -- a capped
    device is then also timed, in the same synchronised window, on the cliff
    rectangle on the other side of its operating point, so both sides of its
    model get their synchronised level.  ci_permille: the sampling stop rule
    for these timings (option "sample_rel_ci_permille"; restored to Q8's 25
    afterwards) -- a level ratio carries its sample's noise into the partition."""
    if ci_permille is not None:
        ctx.set_option("sample_rel_ci_permille", int(ci_permille))
        try:
            return refine(ctx, n, b, models, rounds, arrange, concurrent, dtype, splits, cliffs, log, None)
        finally:
            ctx.set_option("sample_rel_ci_permille", 25)
    T = n * n
    p = len(models)
    base = [(list(xs), list(ss)) for xs, ss in models]   # the size sweep's shapes
    mods = [(list(xs), list(ss)) for xs, ss in models]
    splits = splits or [None] * p
    cliffs = cliffs or [None] * p

    def place(m):
        d = pkg.fpm_partition(T, m)
        r = pkg.colpart_arrange_fpm(n, d, m) if arrange == "fpm" else pkg.colpart_arrange(n, d)
        return d, r

    d, rects = place(mods)
    placed_by = [(list(xs), list(ss)) for xs, ss in mods]   # the models this candidate was placed with
    hist = []
    best = None   # (measured makespan, d, rects, models): the best partition actually timed
    for it in range(rounds):
        shapes = []
        for i, r in enumerate(rects):
            op = (max(1, r[3]), max(1, r[4]))
            other = op
            if splits[i] is not None and cliffs[i] is not None and r[3] * r[4] > 0:
                other = cliffs[i][1] if r[3] * r[4] <= splits[i] else cliffs[i][0]
            shapes.append([op, other])
        if concurrent:
            sp, _, _ = ctx.sample_rects(-1, b, shapes, dtype)
        else:
            sp = [ctx.sample_rects(i, b, shapes[i], dtype)[0] for i in range(p)]
        ratios = []
        for i, r in enumerate(rects):
            x = r[3] * r[4]
            if x <= 0:
                ratios.append(None)
                continue
            xs, ss, k = rescale(base[i], x, sp[i][0], splits[i])
            if splits[i] is not None and shapes[i][1] != shapes[i][0]:   # the other side of the cliff
                xo = shapes[i][1][0] * shapes[i][1][1]
                xs, ss, k2 = rescale((xs, ss), xo, sp[i][1], splits[i])
                ratios.append((k, k2))
            else:
                ratios.append(k)
            mods[i] = (xs, ss)
        # this candidate's makespan as measured in the synchronised window (a run's time is
        # proportional to area / speed at the operating point)
        span = max((r[3] * r[4]) / sp[i][0] for i, r in enumerate(rects) if r[3] * r[4] > 0)
        if best is None or span < best[0]:
            best = (span, list(d), list(rects), placed_by)
        hist.append({"round": it, "d": list(d), "areas": [r[3] * r[4] for r in rects],
                     "sampled_gflops": [v[0] / 1e9 for v in sp], "level_ratio": ratios,
                     "measured_makespan_rel": span})
        d_new, rects_new = place(mods)
        if log:
            log(f"refine {it}: d={d} -> {d_new}  ratios={ratios}")
        if d_new == d:   # converged: the partition the corrected models place is the one just timed
            return mods, hist, d, rects
        d, rects = d_new, rects_new
        placed_by = [(list(xs), list(ss)) for xs, ss in mods]
    # not converged within `rounds` (e.g. oscillating across a memory cliff): the best
    # partition that was actually timed, with the models that placed it
    _, d, rects, m = best
    return m, hist, d, rects
