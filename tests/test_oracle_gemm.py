"""Pins for the oracle GEMM (O5) against what mathematics fixes (not against itself).

* textbook 2x2 worked product (tests/golden/gemm_2x2.txt);
* A . I = A bit-exactly;
* integer matrices: exact product computed independently with Python ints;
* random U[-1,1): numpy/BLAS float64 product (a library routine) within 1e-13;
* non-square / transposed-operand detection (a transposed B must fail).
"""
import os

import numpy as np
import pytest

import synth
from oracle import gemm as og

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "gemm_2x2.txt")


def _read_golden():
    blocks, cur = [], []
    for line in open(GOLDEN):
        line = line.strip()
        if line.startswith("#"):
            continue
        if not line:
            if cur:
                blocks.append(cur)
                cur = []
            continue
        cur.append([float(v) for v in line.split()])
    if cur:
        blocks.append(cur)
    return [np.array(b) for b in blocks]


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_textbook_2x2(dt):
    A, B, C = _read_golden()
    out = og.gemm(A.astype(dt), B.astype(dt))
    assert np.array_equal(out, C)


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_identity_exact(dt):
    A = synth.matrix_pm1(11, 67, dtype=dt)
    I = np.eye(67, dtype=dt)
    assert np.array_equal(og.gemm(A, I), A.astype(np.float64))
    assert np.array_equal(og.gemm(I, A), A.astype(np.float64))


def test_integer_exact_against_python_ints():
    N = 40
    A = synth.matrix_int(3, N)
    B = synth.matrix_int(4, N)
    Ai = [[int(v) for v in row] for row in A]
    Bi = [[int(v) for v in row] for row in B]
    ref = [[sum(Ai[i][k] * Bi[k][j] for k in range(N)) for j in range(N)] for i in range(N)]
    assert np.array_equal(og.gemm(A, B), np.array(ref, dtype=np.float64))


def test_nonsquare_against_blas():
    rng = np.random.default_rng(5)
    A = rng.uniform(-1, 1, size=(37, 129))
    B = rng.uniform(-1, 1, size=(129, 53))
    ref = A @ B
    out = og.gemm(A, B)
    assert np.max(np.abs(out - ref)) <= 1e-13 * np.max(np.abs(ref))
    # a transposed operand must be caught (the product is not symmetric)
    Asq = rng.uniform(-1, 1, size=(32, 32))
    Bsq = rng.uniform(-1, 1, size=(32, 32))
    assert og.rel_fro(og.gemm(Asq, Bsq.T.copy()), Asq @ Bsq) > 1e-2


def test_random_pm1_f32_vs_blas():
    N = 96
    A = synth.matrix_pm1(1, N)
    B = synth.matrix_pm1(2, N)
    ref = A.astype(np.float64) @ B.astype(np.float64)
    assert og.rel_fro(og.gemm(A, B), ref) < 1e-14


def test_rel_fro_definition():
    ref = np.array([[3.0, 0.0], [0.0, 4.0]])
    test = np.array([[3.0, 0.0], [0.0, 4.5]])
    assert og.rel_fro(test, ref) == pytest.approx(0.5 / 5.0, rel=0, abs=1e-16)
