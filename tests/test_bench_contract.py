"""bench.py contract checks that run without a GPU: the reference arm (the CPU
oracle on a bounded sample) prints one JSON line with the required keys, and a
non-zero rank under torchrun prints nothing."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None):
    e = dict(os.environ)
    e.update(env or {})
    out = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                         cwd=ROOT, env=e, timeout=300)
    assert out.returncode == 0, out.stderr
    return [l for l in out.stdout.splitlines() if l.strip()]


def test_reference_arm_json_line():
    lines = _run(["--impl", "reference", "--N", "2048", "--b", "1024", "--steps", "2", "--warmup", "1"])
    assert len(lines) == 1
    d = json.loads(lines[0])
    for key in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
                "scaling", "vs_baseline", "dtype", "data", "config", "cpu_baseline", "e2e", "impl"):
        assert key in d, key
    assert d["impl"] == "reference" and d["value"] > 0 and d["steps"] == 2
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["cores"] >= 1
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["e2e"]["d2h_bytes_per_step"] == 0
    assert d["config"]["N"] == 2048


def test_reference_arm_nonzero_rank_is_silent():
    lines = _run(["--impl", "reference", "--N", "2048", "--steps", "1", "--warmup", "0"],
                 env={"RANK": "1", "WORLD_SIZE": "1"})
    assert lines == []


@__import__("pytest").mark.gpu
def test_ours_json_line_contract_gpu():
    """The GPU arm at a small size prints one JSON line with the contract's keys:
    roofline (bound / achieved / peak / unit / frac / traffic), cpu_baseline,
    e2e with the copied bytes, gpu_launches > 0 and the clocks record."""
    import pytest
    torch = pytest.importorskip("torch")
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    lines = _run(["--N", "8192", "--b", "1024", "--steps", "2", "--warmup", "3", "--no-hetero", "--e2e-steps", "1"])
    assert len(lines) == 1
    d = json.loads(lines[0])
    for key in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
                "scaling", "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e",
                "gpu_launches", "clocks"):
        assert key in d, key
    assert d["value"] > 0 and d["n_gpus"] == 1 and d["steps"] == 2 and d["warmup"] == 3
    r = d["roofline"]
    assert r["bound"] == "tensor" and r["unit"] == "TFLOP/s" and 0 < r["frac"] == r["achieved"] / r["peak"]
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 2 * 8192 * 8192 * 4
    assert d["e2e"]["d2h_bytes_per_step"] == 8192 * 8192 * 4
    assert d["gpu_launches"] > 0 and d["cpu_baseline"]["kind"] == "oracle"
    assert "sm_mhz" in d["clocks"] and "reasons" in d["clocks"]


def _bench_module():
    import importlib.util
    spec = importlib.util.spec_from_file_location("bench_mod", os.path.join(ROOT, "bench.py"))
    m = importlib.util.module_from_spec(spec)
    spec.loader.exec_module(m)
    return m


def test_n_gt_1_line_contract():
    """The line bench.py prints at N > 1 (built by its pure build_line from the
    gathered per-device records, as under torchrun): whole-job value = 2 N^3 K /
    sum of max-over-ranks step times, n_gpus = world, strong scaling, per-device
    records, measured and predicted imbalance over the ranks."""
    bm = _bench_module()
    cfg = dict(bm.CONFIGS["c3"])
    N, b = cfg["N"], cfg["b"]
    rects = [[0, 0, 0, 16, 32], [0, 16, 0, 16, 32]]   # p = 2: one column of two 16 x 32-block strips
    per_dev = [{"rank": r, "device": r, "rect": rects[r], "area": 512, "sm_cap": None,
                "compute_s": t, "update_s": 0.9 * t, "span_s": sp, "predicted_s": 0.01}
               for r, (t, sp) in enumerate(((0.010, 0.0100), (0.011, 0.0104)))]
    roof = {"bound": "tensor", "achieved": 400.0, "peak": 464.5, "unit": "TFLOP/s", "frac": 400.0 / 464.5,
            "traffic": None}
    line = bm.build_line(world=2, steps=3, warmup=3, step_times=[0.011, 0.012, 0.011], workload="c3",
                         cfg=cfg, scheme="f16x3", roofline=roof, per_dev=per_dev,
                         e2e={"value": 1.0, "unit": "GFLOP/s", "h2d_bytes_per_step": 1, "d2h_bytes_per_step": 1},
                         cpu=None, parity=None, launches=10, clocks={"sm_mhz": 1.0, "reasons": []},
                         extra_config={"exchange_staging_overlap": [0.9, 0.8]})
    for key in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step", "higher_is_better",
                "scaling", "vs_baseline", "dtype", "data", "config", "roofline", "cpu_baseline", "e2e",
                "gpu_launches", "clocks"):
        assert key in line, key
    assert line["n_gpus"] == 2 and line["scaling"] == "strong" and line["cpu_baseline"] is None
    assert abs(line["value"] - 2.0 * N ** 3 * 3 / 0.034 / 1e9) < 1e-6 * line["value"]
    assert abs(line["ms_per_step"] - 1e3 * 0.034 / 3) < 1e-9
    c = line["config"]
    assert c["p"] == 2 and len(c["per_device"]) == 2 and c["partition"] == [512, 512]
    assert abs(c["imbalance_pct_measured"] - 100.0 * (0.0104 / 0.0102 - 1)) < 1e-9      # finish times
    assert abs(c["imbalance_pct_compute_sum"] - 100.0 * (0.011 / 0.0105 - 1)) < 1e-9
    assert c["imbalance_pct_predicted"] == 0.0
    assert c["exchange_staging_overlap"] == [0.9, 0.8]
    assert line["dtype"].startswith("f32 (F16X3")
    json.dumps(line)


def test_n_gt_1_rank_parity_blocks():
    """N > 1: each rank checks sampled blocks of ITS rectangle of the e2e output
    (host window at rows R0.., columns C0..) against the oracle.  A window equal
    to the exact product passes; a perturbed element in the centre block or an
    off-by-one window offset is caught."""
    import numpy as np

    import synth
    from oracle import gemm as og
    bm = _bench_module()
    N, seeds = 320, (11, 12)
    R0, C0, H, W = 64, 128, 192, 160
    A = synth.rect(seeds[0], N, R0, 0, H, N)
    B = synth.rect(seeds[1], N, 0, C0, N, W)
    hC = og.gemm(A, B).astype(np.float32)
    blocks = bm.e2e_parity_rank(N, hC, (R0, C0, H, W), seeds, rank=1)
    assert [b["block"] for b in blocks] == ["top-left", "bottom-right", "centre"]
    assert blocks[1]["rows"] == [R0 + H - 64, R0 + H] and blocks[1]["cols"] == [C0 + W - 64, C0 + W]
    assert all(b["rank"] == 1 and b["rel_fro"] <= 1e-7 for b in blocks)
    bad = hC.copy()
    bad[(H - 64) // 2 + 5, (W - 64) // 2 + 7] += 1.0
    assert bm.e2e_parity_rank(N, bad, (R0, C0, H, W), seeds, 1)[2]["rel_fro"] > 1e-5
    shifted = bm.e2e_parity_rank(N, hC, (R0 + 1, C0, H, W), seeds, 1)
    assert max(b["rel_fro"] for b in shifted) > 1e-2
