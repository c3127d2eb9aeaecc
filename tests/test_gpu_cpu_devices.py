"""Mixed host-CPU + GPU contexts (§VI: the hybrid partition of
sockets and GPUs, "22 CPU cores and 2 GPUs"): the CPU
devices' rectangles are updated by their host GEMM on pinned cores while the
GPU devices run their tcgen05 updates; pivots cross between them (GPU staging
kernels read CPU devices' mapped host memory, CPU devices pull GPU-held pivots
device -> host).  C vs the oracle, partitions and arrangements bit-exact."""
import numpy as np
import pytest

import synth
from oracle import fpm as ofpm
from oracle import gemm as og

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

CPU = pkg.FPM_CPU_DEVICE


@pytest.fixture(autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    yield


def _cores(k):
    n = len(pkg.cpu_cores()) - 1       # the first core drives the GPUs
    if n < k:
        pytest.skip(f"needs {k + 1} host cores")
    return k


@pytest.mark.parametrize("dt,tol", [(pkg.FPM_F32, 1e-5), (pkg.FPM_F64, 1e-12)])
@pytest.mark.parametrize("d", [[50, 14], [14, 50], [30, 20, 14]])
def test_mixed_run_parity(dt, tol, d):
    """pmm_run on [GPU, CPU(, CPU)]: every device takes pivots from the others
    (arrangements where a CPU device shares a column with a GPU device)."""
    N, b = 512, 64
    n = N // b
    devs = [0] + [CPU] * (len(d) - 1)
    _cores(2 * (len(d) - 1))
    caps = [0] + [2] * (len(d) - 1)
    rects = pkg.colpart_arrange(n, d)
    npdt = np.float32 if dt == pkg.FPM_F32 else np.float64
    A = synth.rect(1, N, 0, 0, N, N).astype(npdt)
    B = synth.rect(2, N, 0, 0, N, N).astype(npdt)
    C = np.full((N, N), np.nan, npdt)
    with pkg.Context.local(devs, sm_caps=caps) as ctx:
        st = ctx.run(A, B, C, N, b, rects, dt)
    assert og.rel_fro(C, og.gemm(A, B)) <= tol
    assert all(st.per_dev_compute_s[i] > 0 for i in range(len(d)))


def test_mixed_integers_exact_resident_and_compute_into():
    """Resident inputs (on-device / on-host synthetic fill by the same
    generator), pmm_compute then pmm_compute_into: integers bit-exact."""
    N, b = 1024, 128
    n = N // b
    rects = pkg.colpart_arrange(n, [30, 20, 8, 6])
    _cores(4)
    with pkg.Context.local([0, 0, CPU, CPU], sm_caps=[74, 60, 2, 2]) as ctx:
        ctx.setup(N, b, rects, pkg.FPM_F32)
        ctx.fill_synthetic(11, 12, pkg.FPM_DIST_INT)
        ctx.compute()
        ref = og.gemm(synth.rect(11, N, 0, 0, N, N, synth.DIST_INT), synth.rect(12, N, 0, 0, N, N, synth.DIST_INT))
        for (_, r0, c0, h, w) in rects:
            R0, C0 = r0 * b, c0 * b
            got = ctx.download_block(R0 + h * b - 8, C0 + w * b - 8, 8, 8)
            np.testing.assert_array_equal(got, ref[R0 + h * b - 8:R0 + h * b, C0 + w * b - 8:C0 + w * b])
        C = np.full((N, N), np.nan, np.float32)
        ctx.compute_into(C, N)
    np.testing.assert_array_equal(C, ref.astype(np.float32))


def test_mixed_fpm_pipeline():
    """The paper's hybrid pipeline: FPMs sampled for a GPU device and
    a CPU socket, FPM partition and arrangement bit-exact with the oracle, the
    multiply within the FP32 tolerance."""
    N, b = 1024, 64
    n = N // b
    sizes = [1, 4, 16, 64, 256]
    with pkg.Context.local([0, CPU], sm_caps=[2, _cores(4)]) as ctx:   # one CTA pair: the socket gets a share
        models = [(sizes, ctx.sample(i, b, sizes, pkg.FPM_F32)[0]) for i in range(2)]
        assert all(s > 0 for _, sp in models for s in sp)
        d = pkg.fpm_partition(n * n, models)
        assert d == ofpm.partition(n * n, models)
        rects = pkg.colpart_arrange(n, d)
        assert rects == ofpm.arrange(n, d)
        A = synth.rect(3, N, 0, 0, N, N)
        B = synth.rect(4, N, 0, 0, N, N)
        C = np.empty((N, N), np.float32)
        ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
    assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5
    assert d[1] > 0 and d[0] > d[1]   # the 2-SM GPU device outruns the 4-core socket, both get work


def test_mixed_context_synchronised_sampling():
    """fpm_sample(dev = -1) on a GPU device + a CPU device: both sampled in step
    (P:10 (ii)), each on its own host thread; the GPU device (8 SMs) outruns a
    2-core socket, and the synchronised speeds stay within 25 % of the
    exclusive ones (this host's GPU / socket contention is small)."""
    with pkg.Context.local([0, CPU], sm_caps=[8, _cores(2)]) as ctx:
        sp, ci, reps = ctx.sample(-1, 256, [16, 64], pkg.FPM_F32)
        assert len(sp) == 2 and all(v > 0 for r in sp for v in r)
        assert sp[0][1] > sp[1][1]
        alone = [ctx.sample(i, 256, [16, 64], pkg.FPM_F32)[0] for i in range(2)]
        for i in range(2):
            assert 0.75 < sp[i][1] / alone[i][1] < 1.33, (i, sp[i][1], alone[i][1])
