"""Seeded synthetic inputs shared by the oracle, the tests and the bench.

This module holds NO arithmetic of the method (no GEMM, no partitioning, no
arrangement).  It only draws reproducible numbers.  Both sides of every parity
check take their inputs from here (or, for the CUDA side at full size, from a
re-implementation of the SAME counter-based generator in
``paper_conf_cluster_zhongrl12_b200/csrc/kernels/synth.cu``):

* ``matrix_pm1``  — i.i.d. U[-1, 1) entries (reading Q16; PAPER.md
  P:15 "For simplicity, we work with square matrices" fixes only the shape).
* ``matrix_int``  — integers in [-8, 8] (exact-arithmetic pins).
* ``random_models`` — random speed functions s(x) sampled at x = m^2 blocks
  ("timing the kernel with the submatrices of size sqrt(x) x sqrt(x)").

Counter-based generator (identical bits on host and device):

    key  = (seed * 0xD1B54A32D192ED03) mod 2^64
    z    = key + (idx + 1) * 0x9E3779B97F4A7C15        (mod 2^64)
    z    = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9
    z    = (z ^ (z >> 27)) * 0x94D049BB133111EB
    z    =  z ^ (z >> 31)                               (splitmix64 finaliser)

``idx`` is the row-major element index ``row * N + col`` in the GLOBAL N x N
matrix, so any rectangle can be generated independently.

    U[-1,1):  u24 = z >> 40 ;  x = u24 * 2^-23 - 1     (exact in fp32)
    int:      x = (z >> 32) % 17 - 8
"""
from __future__ import annotations

import numpy as np

_M64 = (1 << 64) - 1
_GOLD = np.uint64(0x9E3779B97F4A7C15)
_KEYMUL = 0xD1B54A32D192ED03
_MIX1 = np.uint64(0xBF58476D1CE4E5B9)
_MIX2 = np.uint64(0x94D049BB133111EB)

DIST_PM1 = 0   # U[-1, 1)
DIST_INT = 1   # integers in [-8, 8]


def _hash(seed: int, idx: np.ndarray) -> np.ndarray:
    key = np.uint64((int(seed) * _KEYMUL) & _M64)
    with np.errstate(over="ignore"):
        z = key + (idx.astype(np.uint64) + np.uint64(1)) * _GOLD
        z = (z ^ (z >> np.uint64(30))) * _MIX1
        z = (z ^ (z >> np.uint64(27))) * _MIX2
        z = z ^ (z >> np.uint64(31))
    return z


def hash64(seed: int, idx) -> np.ndarray:
    """The raw 64-bit counter hash (exposed for generator-equivalence tests)."""
    return _hash(seed, np.asarray(idx, dtype=np.uint64))


def _indices(N: int, r0: int, c0: int, h: int, w: int) -> np.ndarray:
    rows = np.arange(r0, r0 + h, dtype=np.uint64)[:, None]
    cols = np.arange(c0, c0 + w, dtype=np.uint64)[None, :]
    return rows * np.uint64(N) + cols


def rect(seed: int, N: int, r0: int, c0: int, h: int, w: int, dist: int = DIST_PM1,
         dtype=np.float32) -> np.ndarray:
    """Rows [r0, r0+h) x cols [c0, c0+w) of the seeded global N x N matrix."""
    z = _hash(seed, _indices(N, r0, c0, h, w))
    if dist == DIST_PM1:
        u24 = (z >> np.uint64(40)).astype(np.float64)
        x = u24 * (2.0 ** -23) - 1.0
    elif dist == DIST_INT:
        x = ((z >> np.uint64(32)) % np.uint64(17)).astype(np.float64) - 8.0
    else:
        raise ValueError(f"unknown dist {dist}")
    return x.astype(dtype)


def matrix_pm1(seed: int, N: int, dtype=np.float32) -> np.ndarray:
    return rect(seed, N, 0, 0, N, N, DIST_PM1, dtype)


# Stress distributions for the FP32 parity tests: inputs whose
# magnitudes vary inside a row, which fixed-point-per-row schemes cannot carry.
# Drawn from independent streams of the same counter-based generator.
_STREAM2 = 0x632BE59BD9B4E019
_STREAM3 = 0x8CB92BA72F3D8DD7


def gaussian(seed: int, N: int, r0: int, c0: int, h: int, w: int, dtype=np.float32) -> np.ndarray:
    """N(0, 1) by Box-Muller from two 53-bit uniforms of the element's counter."""
    idx = _indices(N, r0, c0, h, w)
    u1 = ((_hash(seed, idx) >> np.uint64(11)).astype(np.float64) + 1.0) * 2.0 ** -53   # (0, 1]
    u2 = (_hash(seed ^ _STREAM2, idx) >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
    return (np.sqrt(-2.0 * np.log(u1)) * np.cos(2.0 * np.pi * u2)).astype(dtype)


def lognormal_signed(seed: int, N: int, r0: int, c0: int, h: int, w: int, sigma: float = 1.0,
                     dtype=np.float32) -> np.ndarray:
    """Random sign times exp(sigma g), g ~ N(0, 1): magnitudes spread over
    e^(+-4 sigma) inside every row and column."""
    g = gaussian(seed, N, r0, c0, h, w, np.float64)
    sgn = np.where((_hash(seed ^ _STREAM3, _indices(N, r0, c0, h, w)) >> np.uint64(63)) == 0, 1.0, -1.0)
    return (sgn * np.exp(sigma * g)).astype(dtype)


def matrix_int(seed: int, N: int, dtype=np.float32) -> np.ndarray:
    return rect(seed, N, 0, 0, N, N, DIST_INT, dtype)


# Config seeds ("seed 1 for A, seed 2 for B, config index added").
def seeds_for_config(cfg_index: int) -> tuple[int, int]:
    return 1 + cfg_index, 2 + cfg_index


def random_models(rng: np.random.Generator, p: int, npts: int | None = None,
                  monotone_time: bool = True, max_m: int = 12,
                  speed_range=(1.0, 100.0)):
    """Random speed functions as (x[], s[]) pairs, x = m^2 blocks.

    ``monotone_time=True`` draws models whose time t(x) = x / s(x) is
    non-decreasing at the sample points (the shape [5] assumes: a line through
    the origin meets the speed graph once); ``False`` draws arbitrary positive
    speeds, including steep rises that make t(x) locally decreasing.
    """
    models = []
    for _ in range(p):
        n = int(npts if npts is not None else rng.integers(1, 7))
        ms = np.sort(rng.choice(np.arange(1, max_m + 1), size=min(n, max_m), replace=False))
        xs = [int(m * m) for m in ms]
        if monotone_time:
            # pick times t_j non-decreasing, then s_j = x_j / t_j
            base = rng.uniform(*speed_range)
            ts = []
            t_prev = 0.0
            for x in xs:
                t_min = max(t_prev, 1e-12)
                t = max(x / (base * rng.uniform(0.5, 2.0)), t_min * rng.uniform(1.0, 1.5))
                ts.append(t)
                t_prev = t
            ss = [x / t for x, t in zip(xs, ts)]
        else:
            ss = list(rng.uniform(*speed_range, size=len(xs)))
        models.append((xs, [float(s) for s in ss]))
    return models
