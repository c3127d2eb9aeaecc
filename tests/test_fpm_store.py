"""FPM model files (SURVEY §5 checkpoint / resume; P:87 models built in
advance): round trip, stale-metadata refusal, validation, and the partition of
reloaded models bit-exact between the library and the oracle."""
import json

import numpy as np
import pytest

import synth
from oracle import fpm as ofpm

import paper_conf_cluster_zhongrl12_b200 as pkg
from paper_conf_cluster_zhongrl12_b200 import fpm_store as fs

META = dict(device="NVIDIA B200", kind="gpu", sm_cap=30, cores=None, dtype="f32", b=512, scheme="f16x3", fuse=4)


def _recs(rng, p=3):
    out = []
    for i, (xs, ss) in enumerate(synth.random_models(rng, p, npts=5)):
        out.append(fs.record(xs, [s * 1e12 for s in ss], ci=[0.01] * len(xs), reps=[5] * len(xs),
                             **dict(META, sm_cap=10 * (i + 1))))
    return out


def test_round_trip_and_partition_parity(tmp_path):
    rng = np.random.default_rng(3)
    recs = _recs(rng)
    path = str(tmp_path / "fpm.json")
    fs.save(path, recs)
    back = fs.load(path, expect=[{k: r[k] for k in fs.KEYS} for r in recs])
    assert fs.models(back) == fs.models(recs)
    T = 64 * 64
    d = pkg.fpm_partition(T, fs.models(back))
    assert d == ofpm.partition(T, fs.models(back))


def test_stale_file_is_refused(tmp_path):
    recs = _recs(np.random.default_rng(4), p=2)
    path = str(tmp_path / "fpm.json")
    fs.save(path, recs)
    want = [{k: r[k] for k in fs.KEYS} for r in recs]
    want[1]["b"] = 1024                                  # models of another block size
    with pytest.raises(ValueError):
        fs.load(path, expect=want)
    with pytest.raises(ValueError):
        fs.load(path, expect=want[:1])                   # another device count


def test_invalid_points_and_files(tmp_path):
    with pytest.raises(ValueError):
        fs.record([4, 1], [1.0, 2.0], **META)            # x not increasing
    with pytest.raises(ValueError):
        fs.record([1, 4], [1.0, 0.0], **META)            # non-positive speed
    with pytest.raises(ValueError):
        fs.record([1], [1.0], **{k: v for k, v in META.items() if k != "b"})
    bad = tmp_path / "x.json"
    bad.write_text(json.dumps({"format": "other", "devices": []}))
    with pytest.raises(ValueError):
        fs.load(str(bad))
