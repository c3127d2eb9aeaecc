"""B200-native FPM-partitioned column-based parallel matrix multiplication.

Zhong, Rychkov, Lastovetsky, "Data Partitioning on Heterogeneous Multicore and
Multi-GPU Systems Using Functional Performance Models of Data-Parallel
Applications", Cluster 2012.  The application "takes the FPMs of
heterogeneous processors as input, partitions the matrices using the FPM-based
data partitioning algorithm, and performs the blocked matrix multiplication,
using the GEMM kernel".  The Python names mirror the C ABI
(include/fpmpmm.h): ``fpm_sample``, ``fpm_partition``, ``colpart_arrange``,
``pmm_run``.  This module only marshals arguments; the work happens in
``libfpmpmm.so``.
"""
from __future__ import annotations

import ctypes
from typing import List, Sequence, Tuple

from . import _lib
from ._lib import (FPM_CPU_DEVICE, FPM_DIST_INT, FPM_DIST_PM1, FPM_F32, FPM_F64, SCHEME_F16I8, SCHEME_F16X3, SCHEME_TF32X3,  # noqa: F401,E501
                   FpmError, PmmStats, check, lib)

Model = Tuple[Sequence[int], Sequence[float]]
Rect = Tuple[int, int, int, int, int]

__all__ = [
    "fpm_model_speed", "fpm_partition", "colpart_arrange", "colpart_arrange_fpm", "colpart_plan_step", "Context",
    "fpm_sample", "pmm_run", "FpmError", "FPM_F32", "FPM_F64", "FPM_DIST_PM1", "FPM_DIST_INT",
]


# ---------------------------------------------------------- host algorithms
def fpm_model_speed(model: Model, x: int) -> float:
    arr, keep = _lib._models([model])
    out = ctypes.c_double()
    check(lib.fpm_model_speed(arr, int(x), ctypes.byref(out)))
    return out.value


def fpm_partition(total_blocks: int, models: Sequence[Model], return_iters: bool = False):
    """Integer areas d_i, sum d = total_blocks, equal-time under the FPMs (P:9, [5])."""
    p = len(models)
    arr, keep = _lib._models(models)
    d = (ctypes.c_int64 * p)()
    iters = ctypes.c_int32()
    check(lib.fpm_partition(int(total_blocks), p, arr, d, ctypes.byref(iters)))
    out = list(d)
    return (out, iters.value) if return_iters else out


def colpart_arrange(n: int, d: Sequence[int]) -> List[Rect]:
    """Column-based rectangles (col, row0, col0, h, w) in blocks ([17])."""
    p = len(d)
    da = (ctypes.c_int64 * p)(*[int(v) for v in d])
    out = (_lib.ColpartRect * p)()
    check(lib.colpart_arrange(int(n), p, da, out))
    return _lib.rects_from_c(out)


def colpart_arrange_fpm(n: int, d: Sequence[int], models: Sequence[Model]) -> List[Rect]:
    """Column-based rectangles with integer widths / heights chosen on the FPMs
    (min-max predicted time, then half-perimeters; include/fpmpmm.h)."""
    p = len(d)
    da = (ctypes.c_int64 * p)(*[int(v) for v in d])
    arr, keep = _lib._models(models)
    out = (_lib.ColpartRect * p)()
    check(lib.colpart_arrange_fpm(int(n), p, da, arr, out))
    return _lib.rects_from_c(out)


def colpart_plan_step(n: int, rects: Sequence[Rect], k: int):
    """Pivot delivery of iteration k: (a_moves, b_moves) as (src, dst, begin, end)."""
    p = len(rects)
    rc = _lib.rects_to_c(rects)
    cap = p * p + 4
    am = (_lib.ColpartMove * cap)()
    bm = (_lib.ColpartMove * cap)()
    na, nb = ctypes.c_int32(), ctypes.c_int32()
    check(lib.colpart_plan_step(int(n), p, rc, int(k), am, cap, ctypes.byref(na), bm, cap, ctypes.byref(nb)))
    conv = lambda m: (m.src, m.dst, m.begin, m.end)  # noqa: E731
    return [conv(am[i]) for i in range(na.value)], [conv(bm[i]) for i in range(nb.value)]


# ------------------------------------------------------------------ runtime
class Context:
    """Owns a pmm_ctx: devices, streams, resident buffers, NCCL communicators."""

    def __init__(self, handle: int, p: int, local_devices: int = 1):
        self._h = ctypes.c_void_p(handle)
        self.p = p                          # devices of the arrangement
        self.local_devices = local_devices  # devices driven by this process

    @classmethod
    def local(cls, cuda_devices: Sequence[int], sm_caps: Sequence[int] | None = None) -> "Context":
        p = len(cuda_devices)
        devs = (ctypes.c_int32 * p)(*cuda_devices)
        caps = (ctypes.c_int32 * p)(*(sm_caps or [0] * p))
        h = ctypes.c_void_p()
        check(lib.pmm_create_local(p, devs, caps, ctypes.byref(h)))
        return cls(h.value, p, p)

    @staticmethod
    def nccl_unique_id() -> bytes:
        buf = ctypes.create_string_buffer(128)
        check(lib.pmm_nccl_unique_id(buf))
        return buf.raw

    @classmethod
    def nccl(cls, rank: int, world: int, cuda_device: int, nccl_id: bytes, sm_cap: int = 0) -> "Context":
        h = ctypes.c_void_p()
        check(lib.pmm_create_nccl(rank, world, cuda_device, sm_cap, nccl_id, ctypes.byref(h)))
        return cls(h.value, world)

    @classmethod
    def ipc(cls, rank: int, world: int, cuda_device: int, sm_cap: int = 0) -> "Context":
        """One process per GPU, pivots pulled from peers' memory (CUDA IPC)."""
        h = ctypes.c_void_p()
        check(lib.pmm_create_ipc(rank, world, cuda_device, sm_cap, ctypes.byref(h)))
        return cls(h.value, world)

    def ipc_export(self) -> bytes:
        buf = ctypes.create_string_buffer(_lib.FPM_IPC_BLOB_BYTES)
        check(lib.pmm_ipc_export(self._h, buf))
        return buf.raw

    def ipc_import(self, blobs: Sequence[bytes]) -> None:
        joined = b"".join(blobs)
        check(lib.pmm_ipc_import(self._h, joined, len(blobs)))

    def close(self) -> None:
        if self._h:
            check(lib.pmm_destroy(self._h))
            self._h = ctypes.c_void_p()

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def set_option(self, key: str, value: int) -> None:
        check(lib.pmm_set_option(self._h, key.encode(), int(value)))

    def set_device_option(self, dev: int, key: str, value: int) -> None:
        """Per-device knob (include/fpmpmm.h pmm_set_device_option), e.g.
        ``"c_cap_bytes"``: C_i above this size is held out of core."""
        check(lib.pmm_set_device_option(self._h, int(dev), key.encode(), int(value)))

    def setup(self, N: int, b: int, rects: Sequence[Rect], dtype: int = FPM_F32) -> None:
        self._rects = list(rects)
        self._dtype = dtype
        check(lib.pmm_setup(self._h, int(N), int(b), len(rects), _lib.rects_to_c(rects), int(dtype)))

    def upload(self, A, B, ld: int, row_base: int = 0, col_base: int = 0) -> None:
        check(lib.pmm_upload(self._h, _lib._ptr(A), _lib._ptr(B), int(ld), int(row_base), int(col_base)))

    def fill_synthetic(self, seed_a: int, seed_b: int, dist: int = FPM_DIST_PM1) -> None:
        check(lib.pmm_fill_synthetic(self._h, int(seed_a), int(seed_b), int(dist)))

    def compute(self, zero_c: bool = True) -> PmmStats:
        st = PmmStats()
        check(lib.pmm_compute(self._h, 1 if zero_c else 0, ctypes.byref(st)))
        return st

    def compute_into(self, C, ld: int, row_base: int = 0, col_base: int = 0) -> PmmStats:
        """pmm_compute + download of C_i into the host window, the copy
        overlapped with the last updates (include/fpmpmm.h pmm_compute_into)."""
        st = PmmStats()
        check(lib.pmm_compute_into(self._h, _lib._ptr(C), int(ld), int(row_base), int(col_base),
                                   ctypes.byref(st)))
        return st

    def download(self, C, ld: int, row_base: int = 0, col_base: int = 0) -> None:
        check(lib.pmm_download(self._h, _lib._ptr(C), int(ld), int(row_base), int(col_base)))

    def download_block(self, r0: int, c0: int, rows: int, cols: int, out=None):
        import numpy as np
        dt = np.float64 if getattr(self, "_dtype", FPM_F32) == FPM_F64 else np.float32
        if out is None:
            out = np.empty((rows, cols), dtype=dt)
        check(lib.pmm_download_block(self._h, int(r0), int(c0), int(rows), int(cols), _lib._ptr(out),
                                     out.strides[0] // out.itemsize))
        return out

    def group_times(self, dev: int) -> list:
        """[(staging start, staging end, update start, update end)] per update group
        of the last k-loop on device `dev`, seconds after its start (pmm_group_times)."""
        cnt = ctypes.c_int32(0)
        check(lib.pmm_group_times(self._h, int(dev), None, 0, ctypes.byref(cnt)))
        buf = (ctypes.c_double * (4 * cnt.value))()
        check(lib.pmm_group_times(self._h, int(dev), buf, 4 * cnt.value, ctypes.byref(cnt)))
        return [tuple(buf[4 * g: 4 * g + 4]) for g in range(cnt.value)]

    def run(self, A, B, C, N: int, b: int, rects: Sequence[Rect], dtype: int = FPM_F32,
            ld: int | None = None, row_base: int = 0, col_base: int = 0) -> PmmStats:
        st = PmmStats()
        check(lib.pmm_run(self._h, _lib._ptr(A), _lib._ptr(B), _lib._ptr(C), int(N), int(b), len(rects),
                          _lib.rects_to_c(rects), int(dtype), int(N if ld is None else ld), int(row_base),
                          int(col_base), ctypes.byref(st)))
        return st

    def sample(self, dev: int, b: int, sizes: Sequence[int], dtype: int = FPM_F32):
        """Speed points of device `dev`; dev = -1 samples all local devices at once
        and returns lists of per-device lists."""
        n = len(sizes)
        rows = self.local_devices if dev == -1 else 1
        xs = (ctypes.c_int64 * n)(*[int(x) for x in sizes])
        sp = (ctypes.c_double * (n * rows))()
        ci = (ctypes.c_double * (n * rows))()
        reps = (ctypes.c_int32 * (n * rows))()
        check(lib.fpm_sample(self._h, int(dev), int(dtype), int(b), xs, n, sp, ci, reps))
        if dev != -1:
            return list(sp), list(ci), list(reps)
        cut = lambda a: [list(a[i * n:(i + 1) * n]) for i in range(rows)]  # noqa: E731
        return cut(sp), cut(ci), cut(reps)


    def sample_rects(self, dev: int, b: int, shapes, dtype: int = FPM_F32):
        """Speed points on rectangles (include/fpmpmm.h fpm_sample_rects): shapes =
        [(h, w), ...] blocks; dev = -1: one such list per device of the context,
        all sampled at once.  Returns (speeds, ci, reps) (lists per device for -1)."""
        per_dev = shapes if dev == -1 else [shapes]
        n = len(per_dev[0])
        flat = [int(v) for dev_shapes in per_dev for hw in dev_shapes for v in hw]
        rows = len(per_dev)
        arr = (_lib.i64 * len(flat))(*flat)
        sp = (ctypes.c_double * (n * rows))()
        ci = (ctypes.c_double * (n * rows))()
        reps = (ctypes.c_int32 * (n * rows))()
        check(lib.fpm_sample_rects(self._h, int(dev), int(dtype), int(b), arr, n, sp, ci, reps))
        if dev != -1:
            return list(sp), list(ci), list(reps)
        cut = lambda a: [list(a[i * n:(i + 1) * n]) for i in range(rows)]  # noqa: E731
        return cut(sp), cut(ci), cut(reps)


def fpm_sample(ctx: Context, dev: int, b: int, sizes: Sequence[int], dtype: int = FPM_F32):
    """Speed points s(x) = 2 x b^3 / t(x) of the rank-b kernel."""
    return ctx.sample(dev, b, sizes, dtype)


def pmm_run(ctx: Context, A, B, C, N: int, b: int, rects: Sequence[Rect], dtype: int = FPM_F32,
            ld: int | None = None, row_base: int = 0, col_base: int = 0) -> PmmStats:
    """C = A x B with host A, B, C (row-major windows), blocked column-based."""
    return ctx.run(A, B, C, N, b, rects, dtype, ld, row_base, col_base)


# ------------------------------------------------------- kernel-level calls
def _stream(stream) -> int | None:
    if stream is None:
        try:
            import torch
            return torch.cuda.current_stream().cuda_stream
        except Exception:
            return None
    return int(stream)


def k_split_f32(src, ld, rows, K, scheme, hi, lo, inv_scale=None, stream=None):
    check(lib.fpm_k_split_f32(_lib._ptr(src), ld, rows, K, scheme, _lib._ptr(hi), _lib._ptr(lo),
                              _lib._ptr(inv_scale), _stream(stream)))


def k_split_cols_f32(src, ld, K, W, scheme, hi, lo, inv_scale=None, stream=None):
    check(lib.fpm_k_split_cols_f32(_lib._ptr(src), ld, K, W, scheme, _lib._ptr(hi), _lib._ptr(lo),
                                   _lib._ptr(inv_scale), _stream(stream)))


def k_transpose(src, dtype, ld, rows, cols, dst, stream=None):
    check(lib.fpm_k_transpose(_lib._ptr(src), dtype, ld, rows, cols, _lib._ptr(dst), _stream(stream)))


def k_update_f32(a_hi, a_lo, bt_hi, bt_lo, sa, sb, C, M, Nc, K, ldc, scheme=SCHEME_F16X3, cta_group=2,
                 num_sms=0, accumulate=True, variant=-1, stream=None):
    check(lib.fpm_k_update_f32(_lib._ptr(a_hi), _lib._ptr(a_lo), _lib._ptr(bt_hi), _lib._ptr(bt_lo),
                               _lib._ptr(sa), _lib._ptr(sb), _lib._ptr(C), M, Nc, K, ldc, scheme, cta_group,
                               num_sms, 1 if accumulate else 0, variant, _stream(stream)))


def k_prof(op: int):
    """F16I8 MMA-issuer wait counters (fpm_k_prof): op 1 reset + enable, 0 disable,
    2 read -> dict(tmem_wait, operand_wait, issuer, tiles) in cycles summed over CTAs."""
    out = (ctypes.c_uint64 * 4)()
    check(lib.fpm_k_prof(op, out))
    if op == 2:
        return {"tmem_wait": out[0], "operand_wait": out[1], "issuer": out[2], "tiles": out[3]}
    return None


def k_update_f64(A, lda, Bt, C, M, Nc, K, ldc, accumulate=True, stream=None):
    check(lib.fpm_k_update_f64(_lib._ptr(A), lda, _lib._ptr(Bt), _lib._ptr(C), M, Nc, K, ldc,
                               1 if accumulate else 0, _stream(stream)))


def k_fill_synthetic(dst, dtype, ld, seed, N, r0, c0, rows, cols, dist=FPM_DIST_PM1, stream=None):
    check(lib.fpm_k_fill_synthetic(_lib._ptr(dst), dtype, ld, seed, N, r0, c0, rows, cols, dist,
                                   _stream(stream)))


# ------------------------------------------------------- host-CPU devices
def k_cpu_gemm(A, B, C, accumulate: bool = False, threads: int = 1, pin: bool = False,
               M: int | None = None, N: int | None = None, K: int | None = None,
               lda: int | None = None, seg: int = 0, seg_stride: int = 0, ldb: int | None = None,
               ldc: int | None = None) -> None:
    """The CPU devices' GEMM (include/fpmpmm.h fpm_k_cpu_gemm) on host numpy
    arrays: C (+)= A B, FP32 or FP64 (from C's dtype)."""
    import numpy as np
    dt = FPM_F64 if C.dtype == np.float64 else FPM_F32
    M = C.shape[0] if M is None else M
    N = C.shape[1] if N is None else N
    K = B.shape[0] if K is None else K
    lda = (A.strides[0] // A.itemsize) if lda is None else lda
    ldb = (B.strides[0] // B.itemsize) if ldb is None else ldb
    ldc = (C.strides[0] // C.itemsize) if ldc is None else ldc
    check(lib.fpm_k_cpu_gemm(dt, int(M), int(N), int(K), _lib._ptr(A), int(lda), int(seg), int(seg_stride),
                             _lib._ptr(B), int(ldb), _lib._ptr(C), int(ldc), 1 if accumulate else 0, int(threads),
                             1 if pin else 0))


def cpu_isa() -> str:
    buf = ctypes.create_string_buffer(16)
    check(lib.fpm_cpu_isa(buf, 16))
    return buf.value.decode()


def cpu_cores() -> list:
    n = _lib.i32(0)
    check(lib.fpm_cpu_cores(None, 0, ctypes.byref(n)))
    arr = (_lib.i32 * max(1, n.value))()
    check(lib.fpm_cpu_cores(arr, n.value, ctypes.byref(n)))
    return list(arr[:n.value])
