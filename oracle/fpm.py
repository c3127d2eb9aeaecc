"""Oracle: functional performance models, FPM partition, column-based arrangement,
pivot delivery plan.  TEST INFRASTRUCTURE ONLY (see ``oracle/__init__.py``).

Plain Python, plain loops, exact integer arithmetic wherever the quantity is an
integer.  Every function cites the PAPER.md passage (``P:<line>``) it follows and
the DESIGN.md reading (``Q<n>``) taken where the paper is silent.
"""
from __future__ import annotations

from typing import List, Sequence, Tuple

Model = Tuple[Sequence[int], Sequence[float]]     # (x[] in b x b blocks, s[] in flop/s)


# --------------------------------------------------------------------------- O1
def speed(model: Model, x: int) -> float:
    """s(x): speed of a device for a problem of x b x b blocks.

    P:8 "The functional performance model (FPM) represents the processor speed
    by a function of problem size"; P:18 speed functions are built from points
    x = sqrt(x) x sqrt(x) submatrices.  Interpolation is unstated (reading Q4):
    piecewise linear between sample points, constant beyond both ends.  The
    expression order below is fixed (the library must reproduce its bits).
    """
    xs, ss = model
    if x <= xs[0]:
        return float(ss[0])
    if x >= xs[-1]:
        return float(ss[-1])
    j = 0
    while xs[j + 1] <= x:
        j += 1
    return ss[j] + (ss[j + 1] - ss[j]) * float(x - xs[j]) / float(xs[j + 1] - xs[j])


def time(model: Model, x: int) -> float:
    """t(x) = x / s(x): predicted time of x blocks (P:9 "all processors complete
    their work within the same time"; x/s is the time of x units at speed s)."""
    if x == 0:
        return 0.0
    return float(x) / speed(model, x)


def validate_model(model: Model) -> bool:
    """Reading of the FPM data structure: npts >= 1, x strictly
    increasing integers >= 1, s finite and > 0."""
    xs, ss = model
    if len(xs) < 1 or len(xs) != len(ss):
        return False
    for j, x in enumerate(xs):
        if int(x) != x or x < 1:
            return False
        if j and xs[j] <= xs[j - 1]:
            return False
    for s in ss:
        if not (s > 0.0) or s != s or s == float("inf"):
            return False
    return True


# --------------------------------------------------------------------------- O2
def partition(T: int, models: Sequence[Model]) -> List[int]:
    """Canonical FPM partition of T blocks over p devices (reading Q1-Q3).

    P:9: high performance "can be achieved when all processors complete their
    work within the same time"; "the area of each rectangle is proportional
    to the speed of the processor ... given by the speed function of the
    processor for the assigned problem size".  The integer partition that makes
    the times d_i / s_i(d_i) as equal as possible (min-max) is built by giving
    the blocks out one at a time, each to the device that would finish it
    earliest: key (t_i(d_i + 1), i), ties to the lowest index.  For models
    whose time is non-decreasing this is exactly min-max optimal (the
    discrete form of the "line through the origin" solution of [5]).
    """
    p = len(models)
    d = [0] * p
    for _ in range(T):
        best_i = -1
        best_t = 0.0
        for i in range(p):
            t = time(models[i], d[i] + 1)
            if best_i < 0 or t < best_t:
                best_i, best_t = i, t
        d[best_i] += 1
    return d


def makespan(models: Sequence[Model], d: Sequence[int]) -> float:
    """max_i t_i(d_i): the predicted parallel computation time of a partition."""
    return max(time(m, x) for m, x in zip(models, d))


# --------------------------------------------------------------------------- O4
def arrange(n: int, d: Sequence[int]) -> List[Tuple[int, int, int, int, int]]:
    """Column-based 2D arrangement of areas d_i on the n x n block grid.

    P:15: "matrices A, B and C are partitioned over a 2D arrangement of
    heterogeneous processors so that the area of each rectangle is proportional
    to the speed of the processor"; "The partitioning algorithm ... arranges
    the submatrices to be as square as possible, minimising the total volume of
    communications" (algorithm delegated to [17]; reading Q10):

      1. sort devices by (-d_i, i); devices with d_i = 0 get empty rectangles;
      2. enumerate every split of that order into consecutive columns;
      3. cost = sum_j (k_j * A_j + T)  (= n * total half-perimeter with
         fractional widths A_j / n and heights n d_i / A_j);
      4. choose min by (cost, #columns, tuple of column sizes);
      5. widths  = largest-remainder rounding of A_j / n to sum n
         (ties -> lower column index);
      6. heights = largest-remainder rounding of n d_i / A_j to sum n inside the
         column (ties -> earlier in the column);
      7. columns left to right, devices top to bottom in sorted order.

    Returns one (col, row0, col0, h, w) per device, in blocks.
    """
    p = len(d)
    T = n * n
    if sum(d) != T:
        raise ValueError("sum(d) != n*n")
    order = sorted(range(p), key=lambda i: (-d[i], i))
    active = [i for i in order if d[i] > 0]
    q = len(active)

    best_key = None
    best_groups = None
    for mask in range(1 << (q - 1)):
        groups = []
        cur = [active[0]]
        for pos in range(1, q):
            if mask & (1 << (pos - 1)):
                groups.append(cur)
                cur = []
            cur.append(active[pos])
        groups.append(cur)
        cost = 0
        for g in groups:
            A = sum(d[i] for i in g)
            cost += len(g) * A + T
        key = (cost, len(groups), tuple(len(g) for g in groups))
        if best_key is None or key < best_key:
            best_key, best_groups = key, groups

    groups = best_groups
    areas = [sum(d[i] for i in g) for g in groups]
    widths = _largest_remainder([a for a in areas], n, n)

    rects = [(-1, 0, 0, 0, 0)] * p
    col0 = 0
    for j, g in enumerate(groups):
        A = areas[j]
        heights = _largest_remainder([n * d[i] for i in g], A, n)
        row0 = 0
        for i, h in zip(g, heights):
            rects[i] = (j, row0, col0, h, widths[j])
            row0 += h
        col0 += widths[j]
    return rects


def arrange_fpm(n: int, d: Sequence[int], models: Sequence[Model]) -> List[Tuple[int, int, int, int, int]]:
    """Column-based arrangement whose integer widths and heights are chosen on the
    FPMs (reading Q25; SURVEY §8(f) NEXT-4 "in-column FPM re-partition").

    P:9: high performance "can be achieved when all processors complete their
    work within the same time"; rectangles "as square as possible,
    minimising the total volume of communications", with areas given by the
    speed functions.  arrange() rounds the continuous quotas to integers, which
    leaves a rounding imbalance (e.g. 132 vs 128 blocks at n = 32, p = 8).  Here
    the equal-time condition decides the integers directly:

      1. sort devices by (-d_i, i); devices with d_i = 0 get empty rectangles;
      2. for every split of that order into consecutive columns:
           column time T_j(w): heights h_i >= 0, sum n, given one row at a time
             from zero to the device (position m in the column) minimising
             (t_i((h_i + 1) w), m); T_j(w) = max_i t_i(h_i w)  (t(0) = 0);
           widths w_j >= 0, sum n, given one column of blocks at a time from
             zero to the column minimising (T_j(w_j + 1), j);
           makespan = max_j T_j(w_j);
           cost = sum over rectangles of positive area of (h_i + w_j);
      3. choose min by (makespan, cost, #columns, tuple of column sizes);
      4. columns of positive width left to right, numbered 0, 1, ...; devices
         top to bottom in sorted order; a device left with zero area gets the
         empty rectangle (-1, 0, 0, 0, 0) (reading Q11).

    For non-decreasing times both greedy steps are min-max optimal (the
    discrete equal-time solution of P:9 on the column's rows, then on the
    columns' widths), and the family contains arrange()'s rounding, so the
    makespan is never above arrange()'s.
    """
    p = len(d)
    if sum(d) != n * n:
        raise ValueError("sum(d) != n*n")
    order = sorted(range(p), key=lambda i: (-d[i], i))
    active = [i for i in order if d[i] > 0]
    q = len(active)

    def heights(g, w):
        h = [0] * len(g)
        for _ in range(n):
            best_m = -1
            best_t = 0.0
            for m in range(len(g)):
                t = time(models[g[m]], (h[m] + 1) * w)
                if best_m < 0 or t < best_t:
                    best_m, best_t = m, t
            h[best_m] += 1
        return h, max(time(models[g[m]], h[m] * w) for m in range(len(g)))

    col_time = {}   # (first, last, w) -> T_j(w): plain memo, no change to the definition

    def T(g, first, w):
        key = (first, len(g), w)
        if key not in col_time:
            col_time[key] = heights(g, w)[1]
        return col_time[key]

    best_key = None
    best = None
    for mask in range(1 << (q - 1)):
        groups, starts = [], []
        cur, start = [active[0]], 0
        for pos in range(1, q):
            if mask & (1 << (pos - 1)):
                groups.append(cur)
                starts.append(start)
                cur, start = [], pos
            cur.append(active[pos])
        groups.append(cur)
        starts.append(start)
        c = len(groups)
        w = [0] * c
        for _ in range(n):
            best_j = -1
            best_t = 0.0
            for j in range(c):
                t = T(groups[j], starts[j], w[j] + 1)
                if best_j < 0 or t < best_t:
                    best_j, best_t = j, t
            w[best_j] += 1
        makespan = max(T(groups[j], starts[j], w[j]) for j in range(c))
        cost = 0
        hs = []
        for j in range(c):
            h = heights(groups[j], w[j])[0]
            hs.append(h)
            cost += sum(x + w[j] for x in h if x * w[j] > 0)
        key = (makespan, cost, c, tuple(len(g) for g in groups))
        if best_key is None or key < best_key:
            best_key, best = key, (groups, w, hs)

    groups, w, hs = best
    rects = [(-1, 0, 0, 0, 0)] * p
    col0 = 0
    col = 0
    for j, g in enumerate(groups):
        if w[j] == 0:
            continue
        row0 = 0
        for i, h in zip(g, hs[j]):
            if h > 0:
                rects[i] = (col, row0, col0, h, w[j])
            row0 += h
        col0 += w[j]
        col += 1
    return rects


def _largest_remainder(numerators: Sequence[int], denominator: int, total: int) -> List[int]:
    """Round quotas numerators[k] / denominator to integers summing to ``total``
    (Hamilton / largest remainder): floors, then +1 to the largest remainders,
    ties to the lower index."""
    floors = [a // denominator for a in numerators]
    rems = [a % denominator for a in numerators]
    left = total - sum(floors)
    ranked = sorted(range(len(numerators)), key=lambda k: (-rems[k], k))
    out = list(floors)
    for k in ranked[:left]:
        out[k] += 1
    return out


# --------------------------------------------------------------------------- O6
def plan_step(rects, n: int, k: int):
    """Who sends what at iteration k ("At each iteration of the main loop,
    pivot column of matrix A and pivot row of matrix B are broadcast
    horizontally and vertically"; reading Q12 for a column-based arrangement).

    Returns ``(a_moves, b_moves)`` in block units:
      a_moves: sorted list of (src, dst, row_begin, row_end): the devices of the
               column containing block-column k send A(rows, k) to every device
               whose row range overlaps (src == dst is a local use);
      b_moves: sorted list of (src, dst, col_begin, col_end): in every column,
               the device whose rows contain block-row k sends B(k, cols) to
               each device of that column (src == dst is a local use).
    """
    live = [i for i, r in enumerate(rects) if r[3] > 0 and r[4] > 0]
    a_moves, b_moves = [], []
    holders = [q for q in live if rects[q][2] <= k < rects[q][2] + rects[q][4]]
    for i in live:
        _, r0, c0, h, w = rects[i]
        for q in holders:
            _, qr0, _, qh, _ = rects[q]
            lo, hi = max(r0, qr0), min(r0 + h, qr0 + qh)
            if lo < hi:
                a_moves.append((q, i, lo, hi))
        owner = [q for q in live if rects[q][0] == rects[i][0]
                 and rects[q][1] <= k < rects[q][1] + rects[q][3]]
        assert len(owner) == 1
        b_moves.append((owner[0], i, c0, c0 + w))
    return sorted(a_moves), sorted(b_moves)
