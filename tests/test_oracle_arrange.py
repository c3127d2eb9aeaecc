"""Pins for oracle O4 (column-based arrangement) and O6 (pivot delivery plan).

Pins (independent of the oracle's own enumeration):
  * tiling invariants: rectangles disjoint and covering the n x n grid;
  * brute force over EVERY set partition of the devices into columns (not only
    the sorted consecutive splits the oracle enumerates): the chosen continuous
    cost sum_j (k_j A_j + T) is the global minimum ("minimising the total
    volume of communications");
  * the continuous cost equals n x the sum of half-perimeters (exact fractions);
  * special cases: p = 1, p = 2 equal, p = 4 equal (2 x 2), p = 8 equal at
    n = 32 (groups 2,3,3; areas 128/132/120);
  * delivery: simulating the plan on numpy arrays gives every device exactly
    A(rows_i, k) and B(k, cols_i) ("pivot column of matrix A and pivot row
    of matrix B are broadcast horizontally and vertically").
"""
from fractions import Fraction

import numpy as np
import pytest

from oracle import fpm


def _check_tiling(n, d, rects):
    grid = np.full((n, n), -1, dtype=np.int64)
    for i, (col, r0, c0, h, w) in enumerate(rects):
        if d[i] == 0:
            assert h * w == 0
            continue
        assert h >= 0 and w >= 0
        sub = grid[r0:r0 + h, c0:c0 + w]
        assert sub.shape == (h, w)
        assert np.all(sub == -1), "overlap"
        sub[...] = i
    assert np.all(grid >= 0), "uncovered block"
    assert sum(r[3] * r[4] for r in rects) == n * n


def _random_d(rng, n, p):
    T = n * n
    cuts = np.sort(rng.choice(np.arange(1, T), size=p - 1, replace=False)) if p > 1 else []
    pts = [0] + list(cuts) + [T]
    return [int(pts[i + 1] - pts[i]) for i in range(p)]


def test_tiling_invariants_random():
    rng = np.random.default_rng(1)
    for trial in range(300):
        n = int(rng.integers(1, 40))
        p = int(rng.integers(1, min(9, n * n) + 1))
        d = _random_d(rng, n, p)
        rects = fpm.arrange(n, d)
        _check_tiling(n, d, rects)
        cols = {}
        for (col, r0, c0, h, w) in rects:
            if h * w:
                cols.setdefault(col, []).append((r0, c0, h, w))
        assert sum(v[0][3] for v in cols.values()) == n
        for v in cols.values():
            assert sum(h for (_, _, h, _) in v) == n
            assert len({c0 for (_, c0, _, _) in v}) == 1


def _set_partitions(items):
    if not items:
        yield []
        return
    first, rest = items[0], items[1:]
    for part in _set_partitions(rest):
        for k in range(len(part)):
            yield part[:k] + [[first] + part[k]] + part[k + 1:]
        yield [[first]] + part


def _cost(groups, d, T):
    return sum(len(g) * sum(d[i] for i in g) + T for g in groups)


def test_sorted_consecutive_is_globally_optimal():
    rng = np.random.default_rng(2)
    for trial in range(120):
        n = int(rng.integers(3, 30))
        p = int(rng.integers(1, 7))
        d = _random_d(rng, n, p)
        T = n * n
        rects = fpm.arrange(n, d)
        groups = {}
        for i, r in enumerate(rects):
            if d[i] > 0:
                groups.setdefault(r[0], []).append(i)
        chosen = _cost(list(groups.values()), d, T)
        live = [i for i in range(p) if d[i] > 0]
        best = min(_cost(g, d, T) for g in _set_partitions(live))
        assert chosen == best


def test_cost_is_n_times_half_perimeter():
    d = [50, 30, 20]
    n = 10
    groups = [[0], [1, 2]]
    T = n * n
    hp = Fraction(0)
    for g in groups:
        A = sum(d[i] for i in g)
        w = Fraction(A, n)
        for i in g:
            hp += w + Fraction(n * d[i], A)
    assert hp * n == _cost(groups, d, T)


def test_special_cases():
    assert fpm.arrange(7, [49]) == [(0, 0, 0, 7, 7)]
    assert fpm.arrange(8, [32, 32]) == [(0, 0, 0, 4, 8), (0, 4, 0, 4, 8)]
    r4 = fpm.arrange(8, [16, 16, 16, 16])
    assert sorted((r[1], r[2], r[3], r[4]) for r in r4) == [(0, 0, 4, 4), (0, 4, 4, 4), (4, 0, 4, 4), (4, 4, 4, 4)]
    r8 = fpm.arrange(32, [128] * 8)
    sizes = {}
    for r in r8:
        sizes.setdefault(r[0], []).append(r[3] * r[4])
    assert [len(sizes[c]) for c in sorted(sizes)] == [2, 3, 3]
    assert sorted(a for v in sizes.values() for a in v) == [120, 120, 128, 128, 132, 132, 132, 132]
    # zero-area devices get empty rectangles
    rz = fpm.arrange(4, [16, 0])
    assert rz[0] == (0, 0, 0, 4, 4) and rz[1][3] * rz[1][4] == 0


def test_plan_delivers_every_pivot_exactly_once():
    rng = np.random.default_rng(4)
    b = 2
    for trial in range(60):
        n = int(rng.integers(1, 14))
        p = int(rng.integers(1, min(8, n * n) + 1))
        d = _random_d(rng, n, p)
        rects = fpm.arrange(n, d)
        N = n * b
        A = rng.standard_normal((N, N))
        B = rng.standard_normal((N, N))
        # each device stores only its own rectangle of A and B
        loc = {}
        for i, (_, r0, c0, h, w) in enumerate(rects):
            loc[i] = (A[r0 * b:(r0 + h) * b, c0 * b:(c0 + w) * b],
                      B[r0 * b:(r0 + h) * b, c0 * b:(c0 + w) * b])
        for k in range(n):
            a_moves, b_moves = fpm.plan_step(rects, n, k)
            recvA = {i: np.full((rects[i][3] * b, b), np.nan) for i in range(p)}
            recvB = {i: np.full((b, rects[i][4] * b), np.nan) for i in range(p)}
            for (src, dst, lo, hi) in a_moves:
                _, sr0, sc0, _, _ = rects[src]
                piece = loc[src][0][(lo - sr0) * b:(hi - sr0) * b, (k - sc0) * b:(k - sc0 + 1) * b]
                tgt = recvA[dst][(lo - rects[dst][1]) * b:(hi - rects[dst][1]) * b]
                assert np.all(np.isnan(tgt)), "row delivered twice"
                tgt[...] = piece
            for (src, dst, c_lo, c_hi) in b_moves:
                _, sr0, sc0, _, sw = rects[src]
                assert (c_lo, c_hi) == (sc0, sc0 + sw)
                tgt = recvB[dst]
                assert np.all(np.isnan(tgt))
                tgt[...] = loc[src][1][(k - sr0) * b:(k - sr0 + 1) * b, :]
            for i, (_, r0, c0, h, w) in enumerate(rects):
                if h * w == 0:
                    continue
                assert np.array_equal(recvA[i], A[r0 * b:(r0 + h) * b, k * b:(k + 1) * b])
                assert np.array_equal(recvB[i], B[k * b:(k + 1) * b, c0 * b:(c0 + w) * b])


# ------------------------------------------------------------ arrange_fpm (Q25)
import itertools

import synth


def _compositions(total, k):
    """All k-tuples of integers >= 0 summing to total."""
    if k == 1:
        yield (total,)
        return
    for first in range(0, total + 1):
        for rest in _compositions(total - first, k - 1):
            yield (first,) + rest


def _makespan(models, rects):
    return max(fpm.time(models[i], r[3] * r[4]) for i, r in enumerate(rects) if r[3] * r[4] > 0)


def _brute_force_min_makespan(n, d, models):
    """Every split of the (-d_i, i) order into consecutive columns, every
    integer width vector and every integer height vector (all >= 0)."""
    order = [i for i in sorted(range(len(d)), key=lambda i: (-d[i], i)) if d[i] > 0]
    q = len(order)
    best = None
    for mask in range(1 << (q - 1)):
        groups, cur = [], [order[0]]
        for pos in range(1, q):
            if mask & (1 << (pos - 1)):
                groups.append(cur)
                cur = []
            cur.append(order[pos])
        groups.append(cur)
        for ws in _compositions(n, len(groups)):
            worst = 0.0
            for g, w in zip(groups, ws):
                col_best = min(max(fpm.time(models[i], h * w) for i, h in zip(g, hs))
                               for hs in _compositions(n, len(g)))
                worst = max(worst, col_best)
            best = worst if best is None else min(best, worst)
    return best


def test_arrange_fpm_min_max_by_brute_force():
    """For non-decreasing times the greedy widths / heights reach the minimum
    makespan over every integer arrangement of the family (P:9 equal time)."""
    rng = np.random.default_rng(25)
    for trial in range(120):
        n = int(rng.integers(1, 7))
        p = int(rng.integers(1, min(4, n * n) + 1))
        models = synth.random_models(rng, p, monotone_time=True, max_m=4)
        d = fpm.partition(n * n, models)
        if sum(1 for x in d if x > 0) > 3:
            continue
        rects = fpm.arrange_fpm(n, d, models)
        _check_tiling(n, [r[3] * r[4] for r in rects], rects)
        assert _makespan(models, rects) == _brute_force_min_makespan(n, d, models), (n, d, models)


def test_arrange_fpm_never_worse_than_rounding():
    """The same family as arrange(); its rounding is one of the candidates, so
    with non-decreasing times the FPM-chosen integers are never slower."""
    rng = np.random.default_rng(26)
    for trial in range(80):
        n = int(rng.integers(2, 24))
        p = int(rng.integers(1, 7))
        models = synth.random_models(rng, p, monotone_time=True, max_m=24)
        d = fpm.partition(n * n, models)
        r0 = fpm.arrange(n, d)
        r1 = fpm.arrange_fpm(n, d, models)
        _check_tiling(n, [r[3] * r[4] for r in r1], r1)
        assert _makespan(models, r1) <= _makespan(models, r0)


@pytest.mark.parametrize("n,p", [(32, 8), (64, 8), (48, 8), (32, 4), (48, 2)])
def test_arrange_fpm_homogeneous_exact(n, p):
    """Identical devices, p | n: every device gets exactly n^2 / p blocks
    (arrange() leaves 132 / 128 at n = 32, p = 8 and 528 / 512 at n = 64)."""
    models = [([1], [1.0])] * p
    d = fpm.partition(n * n, models)
    rects = fpm.arrange_fpm(n, d, models)
    _check_tiling(n, d, rects)
    assert all(r[3] * r[4] == n * n // p for r in rects)
    assert rects == fpm.arrange_fpm(n, d, models)


def test_arrange_fpm_zero_areas_and_single_device():
    models = [([1], [1.0]), ([1], [2.0]), ([1], [3.0])]
    rects = fpm.arrange_fpm(4, [0, 16, 0], models)
    assert rects == [(-1, 0, 0, 0, 0), (0, 0, 0, 4, 4), (-1, 0, 0, 0, 0)]
    rects = fpm.arrange_fpm(1, [1], [([1], [1.0])])
    assert rects == [(0, 0, 0, 1, 1)]
