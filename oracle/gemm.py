"""ctypes loader for the C oracle GEMM (``oracle/gemm.c``).

TEST INFRASTRUCTURE ONLY (see ``oracle/__init__.py``).  ``build()`` compiles it
with gcc; nothing here touches a GPU or the product library.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "gemm.c")
_LIB = os.path.join(_HERE, "liboracle_gemm.so")
_lib = None


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O2", "-fopenmp", "-fno-fast-math", "-ffp-contract=off",
               "-shared", "-fPIC", "-o", _LIB + ".tmp", _SRC]
        subprocess.check_call(cmd)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        i64, vp = ctypes.c_int64, ctypes.c_void_p
        for name in ("oracle_gemm_f32in", "oracle_gemm_f64in"):
            fn = getattr(lib, name)
            fn.argtypes = [i64, i64, i64, vp, i64, vp, i64, vp, i64]
            fn.restype = None
        lib.oracle_num_threads.restype = ctypes.c_int
        lib.oracle_set_num_threads.argtypes = [ctypes.c_int]
        lib.oracle_set_num_threads.restype = None
        _lib = lib
    return _lib


def num_threads() -> int:
    return int(_load().oracle_num_threads())


def set_num_threads(n: int) -> None:
    """OpenMP threads of the oracle loops (timing only; results do not depend on it)."""
    _load().oracle_set_num_threads(int(n))


def gemm(A: np.ndarray, B: np.ndarray) -> np.ndarray:
    """C = A @ B by the plain triple loop, FP64 accumulation, FP64 result.

    A: (M, K) float32 or float64; B: (K, N) same dtype.  Strided views allowed
    along rows (the inner dimension must be contiguous)."""
    lib = _load()
    if A.dtype != B.dtype or A.dtype not in (np.float32, np.float64):
        raise TypeError("A and B must both be float32 or both float64")
    A = np.ascontiguousarray(A)
    B = np.ascontiguousarray(B)
    M, K = A.shape
    K2, N = B.shape
    if K != K2:
        raise ValueError("inner dimensions differ")
    C = np.empty((M, N), dtype=np.float64)
    fn = lib.oracle_gemm_f32in if A.dtype == np.float32 else lib.oracle_gemm_f64in
    fn(M, N, K, A.ctypes.data, K, B.ctypes.data, N, C.ctypes.data, N)
    return C


def rel_fro(C_test: np.ndarray, C_ref: np.ndarray) -> float:
    """||C_test - C_ref||_F / ||C_ref||_F in FP64 (the north_star tolerance metric)."""
    ref = C_ref.astype(np.float64)
    diff = C_test.astype(np.float64) - ref
    den = np.sqrt(np.sum(ref * ref))
    num = np.sqrt(np.sum(diff * diff))
    return float(num / den) if den > 0 else float(num)
