"""Green-context SM partitions (option "sm_partition" = 1; BASELINE north_star:
heterogeneity emulated by capping SMs per GPU with green contexts): parity of
the whole path with every device confined to its own SMs, and the confinement
itself visible in the speed functions."""
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


@pytest.mark.parametrize("dt,tol", [(pkg.FPM_F32, 1e-5), (pkg.FPM_F64, 1e-12)])
def test_green_partitions_parity(dt, tol):
    N, b = 1024, 64
    n = N // b
    caps = [64, 40, 24, 10]
    d = pkg.fpm_partition(n * n, [([1], [float(c)]) for c in caps])
    rects = pkg.colpart_arrange(n, d)
    npdt = np.float32 if dt == pkg.FPM_F32 else np.float64
    A = synth.rect(1, N, 0, 0, N, N, synth.DIST_PM1, npdt)
    B = synth.rect(2, N, 0, 0, N, N, synth.DIST_PM1, npdt)
    C = np.full((N, N), np.nan, npdt)
    with pkg.Context.local([0] * 4, sm_caps=caps) as ctx:
        ctx.set_option("sm_partition", 1)
        st = ctx.run(A, B, C, N, b, rects, dt)
        assert st.kernel_launches > 0
    assert og.rel_fro(C, og.gemm(A, B)) <= tol


def test_green_integer_exact_with_out_of_core_device():
    N, b = 1024, 128
    n = N // b
    rects = pkg.colpart_arrange(n, [40, 24])
    A = synth.rect(11, N, 0, 0, N, N, synth.DIST_INT)
    B = synth.rect(12, N, 0, 0, N, N, synth.DIST_INT)
    C = np.full((N, N), np.nan, np.float32)
    with pkg.Context.local([0, 0], sm_caps=[96, 48]) as ctx:
        ctx.set_option("sm_partition", 1)
        ctx.set_device_option(1, "c_cap_bytes", 1)
        st = ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
        assert st.ooc_devices == 2
    assert np.array_equal(C.astype(np.float64), og.gemm(A, B))


def test_green_confinement_shows_in_speed():
    """Two devices sampled at once (dev = -1) in disjoint partitions of 96 and
    32 SMs: at a size that fills the GPU the speeds follow the partitions; the
    staging kernels are confined too."""
    with pkg.Context.local([0, 0], sm_caps=[96, 32]) as ctx:
        ctx.set_option("sm_partition", 1)
        sp, _, _ = ctx.sample(-1, 512, [256], pkg.FPM_F32)
        ratio = sp[0][0] / sp[1][0]
        assert 2.0 < ratio < 4.0


def test_green_partition_errors():
    with pkg.Context.local([0, 0], sm_caps=[96, 0]) as ctx:
        with pytest.raises(pkg.FpmError):
            ctx.set_option("sm_partition", 1)           # a device without a cap
    with pkg.Context.local([0, 0], sm_caps=[144, 48]) as ctx:
        with pytest.raises(pkg.FpmError):
            ctx.set_option("sm_partition", 1)           # 192 SMs do not fit one GPU
    with pkg.Context.local([0], sm_caps=[64]) as ctx:
        ctx.set_option("sm_partition", 1)
        ctx.set_option("sm_partition", 0)               # and back to grid caps
        N, b = 256, 64
        A = synth.rect(1, N, 0, 0, N, N)
        B = synth.rect(2, N, 0, 0, N, N)
        C = np.zeros((N, N), np.float32)
        ctx.run(A, B, C, N, b, [(0, 0, 0, 4, 4)], pkg.FPM_F32)
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


@pytest.mark.parametrize("share_b", [1, 0])
@pytest.mark.parametrize("mode", ["compute", "run"])
def test_green_fused_staging_with_shared_b(share_b, mode):
    """In-kernel staging on devices confined to green partitions of one GPU
    (each grid is resident in its own SMs): every update stages its device's
    next group; with share_b a column member stages only its A rows and reads
    the B operand its owner's update staged (the owner's launch waits for the
    members' updates that read its previous B in that slot).  C bit-identical
    to fused_staging = 0, resident and streamed (pmm_run), integer inputs
    bit-exact vs the oracle, repeated calls."""
    N, b = 4096, 256
    n = N // b
    caps = [48, 40, 32]
    rects = pkg.colpart_arrange(n, [120, 80, 56])
    assert len({r[0] for r in rects}) == 2                   # one column holds two devices
    A = synth.rect(11, N, 0, 0, N, N, synth.DIST_INT)
    B = synth.rect(12, N, 0, 0, N, N, synth.DIST_INT)
    out = []
    for fs in (2, 0):
        with pkg.Context.local([0] * 3, sm_caps=caps) as ctx:
            ctx.set_option("sm_partition", 1)
            ctx.set_option("share_b", share_b)
            ctx.set_option("fused_staging", fs)
            C = np.full((N, N), np.nan, np.float32)
            for _ in range(2):
                if mode == "run":
                    ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
                else:
                    ctx.setup(N, b, rects, pkg.FPM_F32)
                    ctx.upload(A, B, N)
                    st = ctx.compute()
                    ctx.download(C, N)
            out.append(C)
    assert np.array_equal(out[0], out[1])
    assert np.array_equal(out[0].astype(np.float64), og.gemm(A, B))
