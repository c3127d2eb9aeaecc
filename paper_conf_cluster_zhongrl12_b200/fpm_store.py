"""FPM model files (SURVEY §5 checkpoint / resume; the speed
functions are "obtained in advance" and reused): one JSON file per set of
devices, each model recorded with what it was measured on, so a run can reuse
models sampled earlier instead of re-sampling, and a stale file (another GPU,
another SM cap, block size, scheme, kernel) is refused rather than silently
used.

    {"format": "fpmpmm-fpm/1",
     "devices": [{"device": "NVIDIA B200", "kind": "gpu" | "cpu", "sm_cap": 30,
                  "cores": null, "dtype": "f32", "b": 512, "scheme": "f16x3",
                  "fuse": 4, "x": [...], "s": [...], "ci": [...], "reps": [...],
                  "sampled_at": "..."}, ...]}

File I/O only: the models themselves come from fpm_sample / fpm_sample_rects
and go to fpm_partition unchanged (x: blocks, s: flop/s).
"""
from __future__ import annotations

import json
import os
import time
from typing import Dict, List, Sequence

FORMAT = "fpmpmm-fpm/1"
KEYS = ("device", "kind", "sm_cap", "cores", "dtype", "b", "scheme", "fuse")


def record(x: Sequence[int], s: Sequence[float], ci: Sequence[float] | None = None,
           reps: Sequence[int] | None = None, **meta) -> Dict:
    """One device's model with its measurement context (meta: the KEYS)."""
    missing = [k for k in KEYS if k not in meta]
    if missing:
        raise ValueError(f"missing metadata {missing}")
    xs = [int(v) for v in x]
    if len(xs) != len(s) or not xs or any(b <= a for a, b in zip(xs, xs[1:])) or xs[0] < 1:
        raise ValueError("x must be strictly increasing positive integers, one speed per point")
    if any(not (v > 0) or v != v or v == float("inf") for v in s):
        raise ValueError("speeds must be finite and > 0")
    rec = {k: meta[k] for k in KEYS}
    rec.update({"x": xs, "s": [float(v) for v in s],
                "ci": None if ci is None else [float(v) for v in ci],
                "reps": None if reps is None else [int(v) for v in reps],
                "sampled_at": meta.get("sampled_at") or time.strftime("%Y-%m-%dT%H:%M:%SZ", time.gmtime())})
    return rec


def save(path: str, records: List[Dict]) -> None:
    """Write atomically (temp file + rename): a reader never sees half a file."""
    os.makedirs(os.path.dirname(os.path.abspath(path)), exist_ok=True)
    tmp = f"{path}.tmp{os.getpid()}"
    with open(tmp, "w") as f:
        json.dump({"format": FORMAT, "devices": records}, f, indent=1)
    os.replace(tmp, path)


def load(path: str, expect: List[Dict] | None = None) -> List[Dict]:
    """Read a model file; with `expect` (one dict of KEYS per device) every
    device's metadata must match, else ValueError (a stale or foreign file)."""
    with open(path) as f:
        doc = json.load(f)
    if doc.get("format") != FORMAT:
        raise ValueError(f"{path}: not an FPM model file ({doc.get('format')!r})")
    recs = doc["devices"]
    for r in recs:   # re-validate the points
        record(r["x"], r["s"], r.get("ci"), r.get("reps"), **{k: r[k] for k in KEYS},
               sampled_at=r.get("sampled_at"))
    if expect is not None:
        if len(expect) != len(recs):
            raise ValueError(f"{path}: {len(recs)} devices, expected {len(expect)}")
        for i, (want, got) in enumerate(zip(expect, recs)):
            diff = {k: (got.get(k), want[k]) for k in KEYS if k in want and got.get(k) != want[k]}
            if diff:
                raise ValueError(f"{path}: device {i} was measured under other conditions: {diff}")
    return recs


def models(records: List[Dict]):
    """The (x, s) pairs fpm_partition takes."""
    return [(r["x"], r["s"]) for r in records]
