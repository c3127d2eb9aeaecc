"""bench.py under torchrun with two ranks on ONE GPU (--same-gpu: the IPC
transport works within a GPU), each config at a reduced size: the N > 1 path
the driver's scaling run takes (IPC mappings, per-rank SM caps in green
partitions for c4, max-over-ranks timing, gathered per-device records, e2e with
per-rank host windows) prints one complete JSON line from rank 0.  The NCCL
transport runs the same with one rank (NCCL forbids two ranks on one GPU)."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    yield


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _torchrun(nproc, args, timeout=600):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py")] + args
    out = subprocess.run(cmd, capture_output=True, text=True, cwd=ROOT, timeout=timeout)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]
    return json.loads(lines[0]), out.stderr


@pytest.mark.parametrize("config,N,b", [("c5", 8192, 1024), ("c3", 4096, 512), ("c4", 4096, 512)])
def test_two_ranks_same_gpu_line(config, N, b):
    d, _ = _torchrun(2, ["--gpus", "2", "--steps", "2", "--warmup", "3", "--same-gpu", "--config", config,
                         "--N", str(N), "--b", str(b), "--e2e-steps", "1", "--hetero-N", "4096"])
    assert d["n_gpus"] == 2 and d["scaling"] == "strong" and d["value"] > 0
    c = d["config"]
    assert c["p"] == 2 and len(c["per_device"]) == 2 and c["transport"] == "ipc"
    assert {x["rank"] for x in c["per_device"]} == {0, 1}
    assert sum(c["partition"]) == (N // b) ** 2
    assert isinstance(c["exchange_staging_overlap"], list) and len(c["exchange_staging_overlap"]) == 2
    assert len(c["exposed_between_updates_ms"]) == 2
    assert d["e2e"]["value"] > 0 and d["e2e"]["h2d_bytes_per_step"] == 2 * N * N * 4
    assert d["roofline"]["frac"] > 0 and d["gpu_launches"] > 0 and d["cpu_baseline"] is None
    # the e2e output of every rank's rectangle checked against the oracle (3 blocks per rank)
    par = d["parity"]
    assert par["ok"] and par["max_rel_fro"] <= 1e-5 and {x["rank"] for x in par["blocks"]} == {0, 1}
    assert len(par["blocks"]) == 6
    ex = c["exchange_roofline"]
    assert ex["bound"] == "nvlink" and ex["peak"] == 900.0 and len(ex["achieved_per_rank"]) == 2
    assert ex["achieved"] > 0 and "same GPU" in ex["path"]
    if config == "c4":
        assert [x["sm_cap"] for x in c["per_device"]] == [144, 128]
        parts = c["partitions"]
        for name in ("fpm", "cpm_ncal", "homogeneous"):
            assert parts[name]["t_s"] > 0 and sum(parts[name]["d"]) == (N // b) ** 2
        assert "hetero" not in d   # the line is itself the heterogeneity run
    else:   # N > 1 lines carry config 4 run across the job's ranks (here at N = 4096)
        h = d["hetero"]
        assert "error" not in h, h
        assert h["N"] == 4096 and h["b"] == 512 and h["sm_caps"] == [144, 128]
        for name in ("fpm", "cpm_ncal", "homogeneous"):
            assert h[name]["t_s"] > 0 and sum(h[name]["d"]) == (4096 // 512) ** 2
            assert h[name]["pct_of_capped_peak"] > 0
        assert h["capped_aggregate_peak_tflops"] > 0 and h["transport"] == "ipc"


def test_nccl_transport_one_rank_line():
    d, err = _torchrun(1, ["--gpus", "1", "--steps", "2", "--warmup", "3", "--config", "c3", "--N", "4096",
                           "--b", "512", "--e2e-steps", "1", "--no-hetero", "--no-cpu-baseline",
                           "--transport", "nccl"])
    assert d["n_gpus"] == 1 and d["value"] > 0 and d["config"]["transport"] == "nccl"
    assert d["e2e"]["value"] > 0
