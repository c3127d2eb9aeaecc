"""ctypes binding of libfpmpmm.so (include/fpmpmm.h).  Argument marshalling only:
every step of the method runs in the library (host algorithms in C++, the
multiply in sm_100a CUDA kernels).  There is no Python or CPU fallback: if the
library is missing, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os
from typing import List, Sequence, Tuple

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libfpmpmm.so")

FPM_OK = 0
FPM_EINVAL = -1
FPM_ENOMEM = -2
FPM_ECUDA = -3
FPM_ENCCL = -4
FPM_EUNSUPPORTED = -5
FPM_ESTATE = -6
FPM_MAX_DEVICES = 16
FPM_IPC_BLOB_BYTES = 256

FPM_F32 = 0
FPM_F64 = 1
FPM_DIST_PM1 = 0
FPM_DIST_INT = 1

SCHEME_F16X3 = 0
SCHEME_TF32X3 = 1
SCHEME_F16I8 = 3      # fp16 main product + int8 cross terms (opt-in: not FP32-class, DESIGN Q15b)
FPM_CPU_DEVICE = -1   # cuda_devices[i] of a host-CPU device (pmm_create_local)

i32, i64, u64, dbl, vp = ctypes.c_int32, ctypes.c_int64, ctypes.c_uint64, ctypes.c_double, ctypes.c_void_p


class FpmModel(ctypes.Structure):
    _fields_ = [("npts", i32), ("x", ctypes.POINTER(i64)), ("s", ctypes.POINTER(dbl))]


class ColpartRect(ctypes.Structure):
    _fields_ = [("col", i32), ("row0", i64), ("col0", i64), ("h", i64), ("w", i64)]


class ColpartMove(ctypes.Structure):
    _fields_ = [("src", i32), ("dst", i32), ("begin", i64), ("end", i64)]


class PmmStats(ctypes.Structure):
    _fields_ = [
        ("t_compute_s", dbl), ("t_upload_s", dbl), ("t_download_s", dbl),
        ("per_dev_compute_s", dbl * FPM_MAX_DEVICES), ("per_dev_update_s", dbl * FPM_MAX_DEVICES),
        ("gflops", dbl), ("imbalance", dbl), ("iters", i64), ("comm_bytes", i64),
        ("kernel_launches", i64), ("updates", i64),
        ("ooc_devices", i64), ("ooc_bytes", i64), ("per_dev_span_s", dbl * FPM_MAX_DEVICES),
    ]

    def as_dict(self, p: int | None = None) -> dict:
        p = FPM_MAX_DEVICES if p is None else p
        return {
            "t_compute_s": self.t_compute_s, "t_upload_s": self.t_upload_s,
            "t_download_s": self.t_download_s,
            "per_dev_compute_s": list(self.per_dev_compute_s[:p]),
            "per_dev_update_s": list(self.per_dev_update_s[:p]),
            "gflops": self.gflops, "imbalance": self.imbalance, "iters": self.iters,
            "comm_bytes": self.comm_bytes, "kernel_launches": self.kernel_launches, "updates": self.updates,
            "ooc_devices": self.ooc_devices, "ooc_bytes": self.ooc_bytes,
            "per_dev_span_s": list(self.per_dev_span_s[:p]),
        }


class FpmError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"[{code}] {msg}")
        self.code = code


if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built: run __graft_entry__.build() (no CPU fallback exists)")

lib = ctypes.CDLL(LIB_PATH)

_SIGS = {
    "fpm_last_error": ([], ctypes.c_char_p),
    "fpm_abi_version": ([], i32),
    "fpm_model_speed": ([ctypes.POINTER(FpmModel), i64, ctypes.POINTER(dbl)], ctypes.c_int),
    "fpm_partition": ([i64, i32, ctypes.POINTER(FpmModel), ctypes.POINTER(i64), ctypes.POINTER(i32)], ctypes.c_int),
    "colpart_arrange": ([i64, i32, ctypes.POINTER(i64), ctypes.POINTER(ColpartRect)], ctypes.c_int),
    "colpart_arrange_fpm": ([i64, i32, ctypes.POINTER(i64), ctypes.POINTER(FpmModel), ctypes.POINTER(ColpartRect)],
                            ctypes.c_int),
    "colpart_plan_step": ([i64, i32, ctypes.POINTER(ColpartRect), i64, ctypes.POINTER(ColpartMove), i32,
                           ctypes.POINTER(i32), ctypes.POINTER(ColpartMove), i32, ctypes.POINTER(i32)],
                          ctypes.c_int),
    "pmm_create_local": ([i32, ctypes.POINTER(i32), ctypes.POINTER(i32), ctypes.POINTER(vp)], ctypes.c_int),
    "pmm_nccl_unique_id": ([ctypes.c_char_p], ctypes.c_int),
    "pmm_create_nccl": ([i32, i32, i32, i32, ctypes.c_char_p, ctypes.POINTER(vp)], ctypes.c_int),
    "pmm_create_ipc": ([i32, i32, i32, i32, ctypes.POINTER(vp)], ctypes.c_int),
    "pmm_ipc_export": ([vp, ctypes.c_char_p], ctypes.c_int),
    "pmm_ipc_import": ([vp, ctypes.c_char_p, i32], ctypes.c_int),
    "pmm_destroy": ([vp], ctypes.c_int),
    "pmm_set_option": ([vp, ctypes.c_char_p, i64], ctypes.c_int),
    "pmm_compute_into": ([vp, vp, i64, i64, i64, ctypes.POINTER(PmmStats)], ctypes.c_int),
    "pmm_set_device_option": ([vp, i32, ctypes.c_char_p, i64], ctypes.c_int),
    "pmm_setup": ([vp, i64, i64, i32, ctypes.POINTER(ColpartRect), ctypes.c_int], ctypes.c_int),
    "pmm_upload": ([vp, vp, vp, i64, i64, i64], ctypes.c_int),
    "pmm_fill_synthetic": ([vp, u64, u64, i32], ctypes.c_int),
    "pmm_compute": ([vp, i32, ctypes.POINTER(PmmStats)], ctypes.c_int),
    "pmm_download": ([vp, vp, i64, i64, i64], ctypes.c_int),
    "pmm_download_block": ([vp, i64, i64, i64, i64, vp, i64], ctypes.c_int),
    "pmm_group_times": ([vp, i32, ctypes.POINTER(dbl), i32, ctypes.POINTER(i32)], ctypes.c_int),
    "pmm_run": ([vp, vp, vp, vp, i64, i64, i32, ctypes.POINTER(ColpartRect), ctypes.c_int, i64, i64, i64,
                 ctypes.POINTER(PmmStats)], ctypes.c_int),
    "fpm_sample": ([vp, i32, ctypes.c_int, i64, ctypes.POINTER(i64), i32, ctypes.POINTER(dbl),
                    ctypes.POINTER(dbl), ctypes.POINTER(i32)], ctypes.c_int),
    "fpm_sample_rects": ([vp, i32, ctypes.c_int, i64, ctypes.POINTER(i64), i32, ctypes.POINTER(dbl),
                          ctypes.POINTER(dbl), ctypes.POINTER(i32)], ctypes.c_int),
    "fpm_k_split_f32": ([vp, i64, i64, i64, i32, vp, vp, vp, vp], ctypes.c_int),
    "fpm_k_split_cols_f32": ([vp, i64, i64, i64, i32, vp, vp, vp, vp], ctypes.c_int),
    "fpm_k_transpose": ([vp, i32, i64, i64, i64, vp, vp], ctypes.c_int),
    "fpm_k_update_f32": ([vp, vp, vp, vp, vp, vp, vp, i64, i64, i64, i64, i32, i32, i32, i32, i32, vp],
                         ctypes.c_int),
    "fpm_k_update_f64": ([vp, i64, vp, vp, i64, i64, i64, i64, i32, vp], ctypes.c_int),
    "fpm_k_prof": ([i32, ctypes.POINTER(u64)], ctypes.c_int),
    "fpm_k_fill_synthetic": ([vp, i32, i64, u64, i64, i64, i64, i64, i64, i32, vp], ctypes.c_int),
    "fpm_k_cpu_gemm": ([i32, i64, i64, i64, vp, i64, i64, i64, vp, i64, vp, i64, i32, i32, i32], ctypes.c_int),
    "fpm_cpu_isa": ([ctypes.c_char_p, i32], ctypes.c_int),
    "fpm_cpu_cores": ([ctypes.POINTER(i32), i32, ctypes.POINTER(i32)], ctypes.c_int),
}
for _name, (_args, _res) in _SIGS.items():
    _fn = getattr(lib, _name)
    _fn.argtypes = _args
    _fn.restype = _res

EXPORTED = tuple(_SIGS)


def check(status: int) -> None:
    if status != FPM_OK:
        raise FpmError(status, lib.fpm_last_error().decode(errors="replace"))


# ------------------------------------------------------------------ helpers
def _models(models: Sequence[Tuple[Sequence[int], Sequence[float]]]):
    keep = []
    arr = (FpmModel * len(models))()
    for i, (xs, ss) in enumerate(models):
        xa = (i64 * len(xs))(*[int(v) for v in xs])
        sa = (dbl * len(ss))(*[float(v) for v in ss])
        keep.append((xa, sa))
        arr[i].npts = len(xs)
        arr[i].x = ctypes.cast(xa, ctypes.POINTER(i64))
        arr[i].s = ctypes.cast(sa, ctypes.POINTER(dbl))
    return arr, keep


def rects_to_c(rects) -> ctypes.Array:
    arr = (ColpartRect * len(rects))()
    for i, r in enumerate(rects):
        arr[i].col, arr[i].row0, arr[i].col0, arr[i].h, arr[i].w = (int(v) for v in r)
    return arr


def rects_from_c(arr) -> List[Tuple[int, int, int, int, int]]:
    return [(r.col, r.row0, r.col0, r.h, r.w) for r in arr]


def _ptr(x) -> int | None:
    """Device/host pointer from an int, a torch tensor or a numpy array."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if hasattr(x, "data_ptr"):
        return x.data_ptr()
    if hasattr(x, "ctypes"):
        return x.ctypes.data
    raise TypeError(f"cannot take a pointer of {type(x)}")
