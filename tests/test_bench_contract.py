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
