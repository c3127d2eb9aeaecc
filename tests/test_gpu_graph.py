"""pmm_compute as one captured CUDA graph (option "graph", default on): the
replay gives the same C as the eager k-loop (bit-identical: same kernels, same
order), keeps the per-group timing events, and survives re-setup, option
changes, out-of-core devices and green partitions."""
import numpy as np
import pytest

import synth
from oracle import gemm as og

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402


@pytest.fixture(autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    yield


def _compute(ctx, N, b, rects, dt, graph, seeds=(5, 6)):
    ctx.set_option("graph", graph)
    ctx.setup(N, b, rects, dt)
    ctx.fill_synthetic(*seeds)
    sts = [ctx.compute() for _ in range(3)]      # capture + 2 replays (or 3 eager runs)
    C = np.full((N, N), np.nan, np.float32 if dt == pkg.FPM_F32 else np.float64)
    ctx.download(C, N)
    return C, sts


@pytest.mark.parametrize("dt", [pkg.FPM_F32, pkg.FPM_F64])
@pytest.mark.parametrize("p", [1, 3])
def test_graph_matches_eager_bitwise(dt, p):
    N, b = 1024, 64
    n = N // b
    rects = pkg.colpart_arrange(n, [n * n - 60 * (p - 1)] + [60] * (p - 1))
    with pkg.Context.local([0] * p) as ctx:
        Cg, stg = _compute(ctx, N, b, rects, dt, 1)
        Ce, ste = _compute(ctx, N, b, rects, dt, 0)
    assert np.array_equal(Cg, Ce)
    ref = og.gemm(synth.rect(5, N, 0, 0, N, N, synth.DIST_PM1, Cg.dtype.type),
                  synth.rect(6, N, 0, 0, N, N, synth.DIST_PM1, Cg.dtype.type))
    assert og.rel_fro(Cg, ref) <= (1e-5 if dt == pkg.FPM_F32 else 1e-12)
    for a, e in zip(stg, ste):
        assert a.kernel_launches == e.kernel_launches and a.updates == e.updates
        assert a.comm_bytes == e.comm_bytes
        assert all(a.per_dev_update_s[i] > 0 for i in range(p) if rects[i][3] * rects[i][4] > 0)


def test_graph_with_out_of_core_and_green():
    N, b = 1024, 128
    n = N // b
    rects = pkg.colpart_arrange(n, [40, 24])
    with pkg.Context.local([0, 0], sm_caps=[96, 48]) as ctx:
        ctx.set_option("sm_partition", 1)
        ctx.set_device_option(1, "c_cap_bytes", 1)
        Cg, stg = _compute(ctx, N, b, rects, pkg.FPM_F32, 1, seeds=(11, 12))
        assert all(s.ooc_devices == 2 and s.ooc_bytes == stg[0].ooc_bytes > 0 for s in stg)
        Ce, _ = _compute(ctx, N, b, rects, pkg.FPM_F32, 0, seeds=(11, 12))
    assert np.array_equal(Cg, Ce)


def test_graph_recaptured_after_changes():
    """A new problem, a new option value and new inputs after a replay."""
    with pkg.Context.local([0, 0]) as ctx:
        for N, b, fuse in ((512, 64, 0), (768, 96, 1), (512, 64, 2)):
            n = N // b
            rects = pkg.colpart_arrange(n, [n * n // 2, n * n - n * n // 2])
            ctx.set_option("fuse", fuse)
            for seeds in ((1, 2), (3, 4)):
                ctx.setup(N, b, rects)
                ctx.fill_synthetic(*seeds)
                ctx.compute()
                ctx.compute()
                C = np.zeros((N, N), np.float32)
                ctx.download(C, N)
                ref = og.gemm(synth.rect(seeds[0], N, 0, 0, N, N), synth.rect(seeds[1], N, 0, 0, N, N))
                assert og.rel_fro(C, ref) <= 1e-5


def test_graph_cuts_small_problem_latency():
    """Config 1 shape (N = 512, b = 64, FP64, two devices): the replayed k-loop
    is not slower than the eager one (it is launch-bound)."""
    N, b = 512, 64
    rects = pkg.colpart_arrange(8, [32, 32])
    with pkg.Context.local([0, 0], sm_caps=[96, 48]) as ctx:
        def best(graph):
            ctx.set_option("graph", graph)
            ctx.setup(N, b, rects, pkg.FPM_F64)
            ctx.fill_synthetic(1, 2)
            return min(ctx.compute().t_compute_s for _ in range(20))
        t_eager, t_graph = best(0), best(1)
        print(f"c1 k-loop: eager {t_eager * 1e6:.1f} us, graph {t_graph * 1e6:.1f} us")
    assert t_graph <= 1.1 * t_eager
