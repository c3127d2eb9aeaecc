"""libfpmpmm host algorithms vs the oracle, bit for bit (no GPU needed).

fpm_partition (geometric bisection + exact integer phase) must equal the
oracle's canonical partition; colpart_arrange and colpart_plan_step must equal
the oracle's arrangement and delivery plan exactly.  Also: the library loads and
exports every function include/fpmpmm.h declares.
"""
import os
import re

import numpy as np
import pytest

import paper_conf_cluster_zhongrl12_b200 as pkg
import synth
from oracle import fpm as ofpm

HEADER = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include", "fpmpmm.h")


def test_exports_every_declared_function():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    names = set(re.findall(r"\b((?:fpm|pmm|colpart)_[a-z0-9_]+)\s*\(", text))
    assert len(names) >= 20
    for name in sorted(names):
        assert hasattr(pkg.lib, name), f"{name} not exported"
    assert set(pkg._lib.EXPORTED) >= names


def test_abi_version():
    assert pkg.lib.fpm_abi_version() == 1


# ----------------------------------------------------------- model evaluation
def test_model_speed_bit_exact():
    rng = np.random.default_rng(10)
    for trial in range(300):
        (m,) = synth.random_models(rng, 1, monotone_time=bool(trial % 2), max_m=20)
        for x in list(range(0, 30)) + [int(v) for v in rng.integers(0, 1000, size=20)]:
            assert pkg.fpm_model_speed(m, x) == ofpm.speed(m, x)


def test_model_validation_errors():
    for bad in [([], []), ([0], [1.0]), ([3, 2], [1.0, 1.0]), ([1], [0.0]), ([1], [float("nan")])]:
        with pytest.raises(pkg.FpmError) as e:
            pkg.fpm_partition(4, [bad])
        assert e.value.code == pkg._lib.FPM_EINVAL


# ------------------------------------------------------------------ partition
def _check_partition(T, models):
    got = pkg.fpm_partition(T, models)
    ref = ofpm.partition(T, models)
    assert got == ref, (T, models, got, ref)


def test_partition_bit_exact_random_monotone():
    rng = np.random.default_rng(11)
    for trial in range(5000):
        p = int(rng.integers(1, 9))
        models = synth.random_models(rng, p, monotone_time=True)
        _check_partition(int(rng.integers(0, 70)), models)


def test_partition_bit_exact_random_nonmonotone_and_ties():
    rng = np.random.default_rng(12)
    for trial in range(5000):
        p = int(rng.integers(1, 7))
        models = synth.random_models(rng, p, monotone_time=False, max_m=8,
                                     speed_range=(1.0, 4.0) if trial % 3 == 0 else (1.0, 100.0))
        if trial % 2 == 0:  # integer speeds: many exact time ties
            models = [(xs, [float(round(s)) for s in ss]) for xs, ss in models]
        _check_partition(int(rng.integers(0, 60)), models)


def test_partition_degenerate():
    m = ([1, 4, 9], [2.0, 3.0, 4.0])
    _check_partition(0, [m, m])
    _check_partition(1, [m] * 8)
    _check_partition(100, [m])
    _check_partition(100, [m] * 16)
    # one dominant device, others nearly idle (zero areas)
    _check_partition(7, [([1], [1e6]), ([1], [1.0]), ([1], [1.0])])
    assert pkg.fpm_partition(7, [([1], [1e6]), ([1], [1.0]), ([1], [1.0])]) == [7, 0, 0]


def _sm_capped_models(caps, b=512, xs=None):
    """Speed ~ SMs used: a rank-b kernel on x blocks runs ceil(tiles / caps) waves."""
    xs = xs or [m * m for m in range(1, 33)]
    models = []
    for cap in caps:
        ss = []
        for x in xs:
            tiles = max(1, (x * b * b) // (256 * 256))
            waves = -(-tiles // (cap // 2))
            ss.append(2.0 * x * b ** 3 / (waves * 1e-4))
        models.append((xs, ss))
    return models


@pytest.mark.parametrize("T,caps", [
    (64, [144, 48]),                                        # config 1 (n = 8)
    (1024, [148, 148]), (1024, [148] * 4), (1024, [148] * 8),  # config 3 (n = 32)
    (4096, [144, 128, 112, 96, 80, 64, 48, 32]),            # config 4 (n = 64)
    (2304, [148] * 8),                                      # config 5 (n = 48)
])
def test_partition_config_models(T, caps):
    models = _sm_capped_models(caps)
    _check_partition(T, models)
    d = pkg.fpm_partition(T, models)
    assert sum(d) == T


def test_partition_scaling_invariance():
    rng = np.random.default_rng(13)
    for trial in range(200):
        models = synth.random_models(rng, 5, monotone_time=bool(trial % 2))
        T = int(rng.integers(1, 200))
        d = pkg.fpm_partition(T, models)
        scaled = [(xs, [s * 2.0 ** 17 for s in ss]) for xs, ss in models]
        assert pkg.fpm_partition(T, scaled) == d


def test_partition_large_T_matches_oracle():
    rng = np.random.default_rng(14)
    models = synth.random_models(rng, 8, monotone_time=True, max_m=70)
    _check_partition(4900, models)


# ---------------------------------------------------------------- arrangement
def _random_d(rng, n, p):
    T = n * n
    cuts = np.sort(rng.choice(np.arange(1, T), size=p - 1, replace=False)) if p > 1 else []
    pts = [0] + list(cuts) + [T]
    return [int(pts[i + 1] - pts[i]) for i in range(p)]


def test_arrange_bit_exact_random():
    rng = np.random.default_rng(15)
    for trial in range(3000):
        n = int(rng.integers(1, 80))
        p = int(rng.integers(1, min(12, n * n) + 1))
        d = _random_d(rng, n, p)
        if trial % 5 == 0 and p > 2:  # zero areas
            d[-1] += d[0]
            d[0] = 0
        assert pkg.colpart_arrange(n, d) == ofpm.arrange(n, d)


def test_arrange_p16():
    rng = np.random.default_rng(16)
    d = _random_d(rng, 64, 16)
    assert pkg.colpart_arrange(64, d) == ofpm.arrange(64, d)


def test_arrange_errors():
    with pytest.raises(pkg.FpmError):
        pkg.colpart_arrange(4, [10, 5])           # sum != n^2
    with pytest.raises(pkg.FpmError):
        pkg.colpart_arrange(4, [17, -1])


def test_arrange_config_cases():
    r8 = pkg.colpart_arrange(32, [128] * 8)
    assert r8 == ofpm.arrange(32, [128] * 8)
    assert sorted(r[3] * r[4] for r in r8) == [120, 120, 128, 128, 132, 132, 132, 132]
    assert pkg.colpart_arrange(48, [288] * 8) == ofpm.arrange(48, [288] * 8)


def test_arrange_fpm_bit_exact_random():
    """colpart_arrange_fpm vs oracle arrange_fpm (Q25): same rectangles, bit for
    bit, for monotone and non-monotone models, with zero areas."""
    rng = np.random.default_rng(25)
    for trial in range(400):
        n = int(rng.integers(1, 28))
        p = int(rng.integers(1, min(7, n * n) + 1))
        models = synth.random_models(rng, p, monotone_time=bool(trial % 3), max_m=20)
        d = ofpm.partition(n * n, models) if trial % 4 else _random_d(rng, n, p)
        if trial % 7 == 0 and p > 2:
            d[-1] += d[0]
            d[0] = 0
        assert pkg.colpart_arrange_fpm(n, d, models) == ofpm.arrange_fpm(n, d, models), (n, d)


@pytest.mark.parametrize("caps", [[30, 26, 24, 20, 16, 14, 10, 6], [144, 128, 112, 96, 80, 64, 48, 32]])
def test_arrange_fpm_config_models(caps):
    """c4-shaped models (8 SM-capped devices, n = 64): bit-exact, and the
    predicted makespan never above colpart_arrange's."""
    n = 64
    models = _sm_capped_models(caps)
    d = pkg.fpm_partition(n * n, models)
    r1 = pkg.colpart_arrange_fpm(n, d, models)
    assert r1 == ofpm.arrange_fpm(n, d, models)
    r0 = pkg.colpart_arrange(n, d)
    ms = lambda rs: max(ofpm.time(m, r[3] * r[4]) for m, r in zip(models, rs) if r[3] * r[4] > 0)  # noqa: E731
    assert ms(r1) <= ms(r0)


def test_arrange_fpm_homogeneous_and_errors():
    m8 = [([1], [1.0])] * 8
    r = pkg.colpart_arrange_fpm(32, [128] * 8, m8)
    assert r == ofpm.arrange_fpm(32, [128] * 8, m8)
    assert all(x[3] * x[4] == 128 for x in r)
    with pytest.raises(pkg.FpmError):
        pkg.colpart_arrange_fpm(4, [10, 5], m8[:2])          # sum != n^2
    with pytest.raises(pkg.FpmError):
        pkg.colpart_arrange_fpm(4, [8, 8], [([1], [1.0]), ([2, 1], [1.0, 1.0])])  # bad model
    with pytest.raises(pkg.FpmError):
        pkg.colpart_arrange_fpm(2048, [2048 * 2048], m8[:1])  # n too large


# ----------------------------------------------------------------------- plan
def test_plan_bit_exact_random():
    rng = np.random.default_rng(17)
    for trial in range(300):
        n = int(rng.integers(1, 20))
        p = int(rng.integers(1, min(10, n * n) + 1))
        d = _random_d(rng, n, p)
        rects = ofpm.arrange(n, d)
        for k in range(n):
            a, b = pkg.colpart_plan_step(n, rects, k)
            ra, rb = ofpm.plan_step(rects, n, k)
            assert a == [tuple(x) for x in ra] and b == [tuple(x) for x in rb]


def test_plan_rejects_bad_tiling():
    with pytest.raises(pkg.FpmError):
        pkg.colpart_plan_step(4, [(0, 0, 0, 2, 4), (0, 1, 0, 2, 4)], 0)  # overlapping rows
