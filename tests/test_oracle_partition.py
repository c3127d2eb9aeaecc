"""Pins for oracle O1 (model evaluation) and O2 (FPM partition).

Each pin is something other than the oracle itself:
  * numpy.interp (library routine) for piecewise-linear evaluation;
  * brute-force enumeration of every integer partition for p in {2, 3}, T <= 40
    (the min-max optimum that P:9 "complete their work within the same time"
    asks for);
  * closed forms: identical models -> even split; constant models -> D'Hondt
    highest-averages apportionment computed by the divisor method;
  * exact invariants: sum d = T (area conservation), scaling all speeds by 2^k;
  * the paper's qualitative Table III result: CPM calibrated while
    the GPU fits its memory overloads it; FPM does not.
"""
import itertools
import os

import numpy as np
import pytest

import synth
from oracle import fpm


def _models(seed, p, monotone=True, **kw):
    return synth.random_models(np.random.default_rng(seed), p, monotone_time=monotone, **kw)


# ------------------------------------------------------------------ O1 pins
def test_speed_matches_numpy_interp():
    rng = np.random.default_rng(0)
    for trial in range(200):
        (xs, ss), = _models(trial, 1, monotone=bool(trial % 2))
        for x in range(1, 170):
            ref = float(np.interp(x, xs, ss))
            assert fpm.speed((xs, ss), x) == pytest.approx(ref, rel=1e-14, abs=0)


def test_speed_sample_points_and_ends_exact():
    xs, ss = [4, 9, 25], [10.0, 30.0, 20.0]
    assert fpm.speed((xs, ss), 4) == 10.0
    assert fpm.speed((xs, ss), 9) == 30.0
    assert fpm.speed((xs, ss), 25) == 20.0
    assert fpm.speed((xs, ss), 1) == 10.0        # constant below the first point
    assert fpm.speed((xs, ss), 1000) == 20.0     # constant beyond the last point
    assert fpm.speed((xs, ss), 17) == 25.0       # midpoint of [9, 25]: (30 + 20) / 2
    assert fpm.time((xs, ss), 17) == 17 / 25.0
    assert fpm.time((xs, ss), 0) == 0.0


def test_validate_model():
    assert fpm.validate_model(([1], [1.0]))
    assert not fpm.validate_model(([], []))
    assert not fpm.validate_model(([0], [1.0]))
    assert not fpm.validate_model(([2, 2], [1.0, 1.0]))
    assert not fpm.validate_model(([1, 4], [1.0, -1.0]))
    assert not fpm.validate_model(([1], [float("nan")]))
    assert not fpm.validate_model(([1], [float("inf")]))


# ------------------------------------------------------------------ O2 pins
def _makespan_np(models, d):
    """Independent of the oracle: t_i(x) = x / s_i(x) with s_i from numpy.interp
    (piecewise linear, constant beyond the ends: reading Q4), max over devices."""
    return max((x / float(np.interp(x, xs, ss)) if x > 0 else 0.0) for (xs, ss), x in zip(models, d))


def _brute(T, models):
    """All compositions of T into p parts; returns (min makespan, the partitions
    within 1e-12 of it, the next larger makespan) -- makespans from _makespan_np."""
    p = len(models)
    scored = []
    for head in itertools.product(range(T + 1), repeat=p - 1):
        if sum(head) > T:
            continue
        d = list(head) + [T - sum(head)]
        scored.append((_makespan_np(models, d), d))
    scored.sort(key=lambda t: t[0])
    best = scored[0][0]
    args = [d for ms, d in scored if ms <= best * (1 + 1e-12)]
    nxt = next((ms for ms, _ in scored if ms > best * (1 + 1e-12)), None)
    return best, args, nxt


def test_makespan_matches_independent_evaluation():
    """fpm.makespan = max_i x_i / s_i(x_i) with the speeds evaluated by numpy.interp
    (same piecewise-linear model, different arithmetic: equal to 1e-12)."""
    rng = np.random.default_rng(17)
    for seed in range(200):
        models = _models(seed, 3, max_m=8)
        d = [int(v) for v in rng.integers(0, 80, 3)]
        ref = _makespan_np(models, d)
        assert abs(fpm.makespan(models, d) - ref) <= 1e-12 * max(ref, 1e-300)


@pytest.mark.parametrize("p", [2, 3])
def test_bruteforce_minmax_optimal(p):
    checked_unique = 0
    for seed in range(60 if p == 2 else 25):
        models = _models(1000 * p + seed, p, max_m=6)
        T = 1 + (seed * 7) % 40
        d = fpm.partition(T, models)
        assert sum(d) == T
        best, args, nxt = _brute(T, models)
        assert _makespan_np(models, d) <= best * (1 + 1e-12)
        # a unique optimum, clearly separated from the runner-up: the partition is it
        if len(args) == 1 and (nxt is None or nxt > best * (1 + 1e-9)):
            assert d == args[0]
            checked_unique += 1
    assert checked_unique > 5


def test_identical_models_even_split():
    for p in range(1, 9):
        for T in (1, 7, 64, 100):
            models = [([1, 4, 9], [3.0, 5.0, 6.0])] * p
            d = fpm.partition(T, models)
            assert d == [T // p + (1 if i < T % p else 0) for i in range(p)]


def _dhondt(T, consts):
    """Highest averages (Jefferson/D'Hondt) by the divisor method: seat i gets
    #{m >= 1 : c_i / m >= lambda*}, lambda* the T-th largest quotient."""
    quot = sorted(((c / m, i) for i, c in enumerate(consts) for m in range(1, T + 1)),
                  reverse=True)
    lam = quot[T - 1][0]
    return [sum(1 for m in range(1, T + 1) if c / m >= lam) for c in consts]


def test_constant_models_are_dhondt():
    rng = np.random.default_rng(3)
    for trial in range(40):
        p = int(rng.integers(2, 9))
        consts = list(rng.uniform(1.0, 50.0, size=p))
        T = int(rng.integers(1, 300))
        d = fpm.partition(T, [([1], [c]) for c in consts])
        assert d == _dhondt(T, consts)


def test_scaling_invariance():
    for seed in range(30):
        models = _models(seed, 4, monotone=bool(seed % 2))
        T = 50 + seed
        d = fpm.partition(T, models)
        for k in (-7, 3, 20):
            scaled = [(xs, [s * 2.0 ** k for s in ss]) for xs, ss in models]
            assert fpm.partition(T, scaled) == d


def test_exchange_certificate_monotone():
    """No block can move to another device and finish earlier (P:9)."""
    for seed in range(50):
        models = _models(500 + seed, 5)
        T = 200
        d = fpm.partition(T, models)
        for i in range(5):
            if d[i] == 0:
                continue
            for j in range(5):
                if j != i:
                    assert fpm.time(models[i], d[i]) <= fpm.time(models[j], d[j] + 1)


def test_zero_blocks_and_single_device():
    assert fpm.partition(0, [([1], [1.0]), ([1], [2.0])]) == [0, 0]
    assert fpm.partition(17, [([1, 4], [1.0, 3.0])]) == [17]


# ---- paper-shaped qualitative pin (Table III; Fig. 6/7)
def _paper_like_models():
    """G1 fast while its share fits (~9x a socket), 6-4x beyond; G2 ~2x;
    sockets S5 = 5/6 S6 (five active cores).  x in 640x640 blocks."""
    s6 = 1.0
    xs = [1, 100, 400, 900, 1089, 1296, 1600, 2500, 3600, 4900]
    g1 = [9.0, 9.0, 9.0, 9.0, 9.0, 6.0, 5.2, 4.6, 4.3, 4.0]
    g2 = [2.0] * len(xs)
    return [(xs, g1), (xs, g2), ([1], [5 / 6 * s6]), ([1], [5 / 6 * s6]),
            ([1], [s6]), ([1], [s6])]


def test_paper_memory_cliff_cpm_overloads_gpu():
    golden = os.path.join(os.path.dirname(__file__), "golden", "table3_paper.txt")
    paper = {}
    for line in open(golden):
        if line.startswith("#") or not line.strip():
            continue
        kind, n, g1, g2, s5, s6 = line.split()
        paper[(kind, int(n))] = (int(g1), int(g2), int(s5), int(s6))
    n = 70
    T = n * n
    models = _paper_like_models()
    d_fpm = fpm.partition(T, models)
    # CPM: constants = speeds measured while the GPU share fits its memory
    cpm_consts = [fpm.speed(m, 400) for m in models]
    d_cpm = fpm.partition(T, [([1], [c]) for c in cpm_consts])
    r_fpm = d_fpm[0] / d_fpm[4]
    r_cpm = d_cpm[0] / d_cpm[4]
    # paper, 70x70: G1/S6 = 2848/366 ~ 7.8 under CPM ("nearly 8"), 2250/504 ~ 4.5 under FPM
    p_cpm = paper[("CPM", 70)][0] / paper[("CPM", 70)][3]
    p_fpm = paper[("FPM", 70)][0] / paper[("FPM", 70)][3]
    assert p_cpm > p_fpm                      # the paper's direction
    assert r_cpm > 7.5 and 3.5 < r_fpm < 6.5  # reproduced with synthetic FPMs
    assert fpm.makespan(models, d_fpm) < fpm.makespan(models, d_cpm)
