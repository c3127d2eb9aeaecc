"""Download-overlapped tail (option "e2e_tail"; pmm_run / pmm_compute_into):
the last update groups run band-major so C_i leaves the device band by band
under the remaining updates.  Same sums per element, so parity with the oracle
(bit-exact on integers) for every tail length, with resident and out-of-core
devices mixed, through pmm_run and pmm_compute_into."""
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


@pytest.mark.parametrize("tail_fuse", [1, 0])
@pytest.mark.parametrize("tail", [-1, 0, 1, 3, 16])
@pytest.mark.parametrize("p", [1, 3])
def test_run_with_tail_parity(tail, p, tail_fuse):
    N, b = 2304, 96                  # n = 24 pivots, fused groups of 8 (K = 768); rects > 2048 rows: 2+ bands
    n = N // b
    rects = pkg.colpart_arrange(n, [n * n - 100 * (p - 1)] + [100] * (p - 1))
    A = synth.rect(1, N, 0, 0, N, N)
    B = synth.rect(2, N, 0, 0, N, N)
    C = np.full((N, N), np.nan, np.float32)
    with pkg.Context.local([0] * p) as ctx:
        ctx.set_option("e2e_tail", tail)
        ctx.set_option("tail_fuse", tail_fuse)
        st = ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
        assert st.updates >= 1
    assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


@pytest.mark.parametrize("scheme", [-1, pkg.SCHEME_F16X3, pkg.SCHEME_TF32X3])   # -1: the default (auto)
def test_fused_tail_common_scale_over_groups(scheme):
    """Fused tail: every row / column takes ONE F16X3 scale over all tail pivots
    (maxima merged across groups and holders).  Block-columns of A and
    block-rows of B scaled by 2^(+-6): a scale taken from one group alone
    would overflow fp16 on another (|x| 2^s > 65504).  (A spread of 2^24 along
    K would push the small values' lo halves into fp16 subnormals: DESIGN.md
    Q15, the limit of one scale per row.)"""
    N, b = 1536, 64
    n = N // b
    rects = pkg.colpart_arrange(n, [300, 160, 116])   # 3 devices, A slices pulled in pieces
    A = synth.rect(3, N, 0, 0, N, N)
    B = synth.rect(4, N, 0, 0, N, N)
    for k in range(n):
        A[:, k * b:(k + 1) * b] *= np.float32(2.0 ** (6 * ((k % 3) - 1)))
        B[k * b:(k + 1) * b, :] *= np.float32(2.0 ** (-6 * ((k % 3) - 1)))
    C = np.full((N, N), np.nan, np.float32)
    with pkg.Context.local([0] * 3) as ctx:
        ctx.set_option("f32_scheme", scheme)
        ctx.set_option("fuse", 2)
        ctx.set_option("e2e_tail", 6)
        ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
    assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


@pytest.mark.parametrize("tail_fuse", [1, 0])
@pytest.mark.parametrize("fuse", [1, 2])
def test_tail_integer_exact_mixed_ooc(fuse, tail_fuse):
    N, b = 1536, 128
    n = N // b
    rects = pkg.colpart_arrange(n, [80, 40, 24])
    A = synth.rect(11, N, 0, 0, N, N, synth.DIST_INT)
    B = synth.rect(12, N, 0, 0, N, N, synth.DIST_INT)
    C = np.full((N, N), np.nan, np.float32)
    with pkg.Context.local([0, 0, 0]) as ctx:
        ctx.set_option("fuse", fuse)
        ctx.set_option("tail_fuse", tail_fuse)
        ctx.set_option("e2e_tail", 4)
        ctx.set_device_option(1, "c_cap_bytes", 1)   # device 1 out of core: no tail, copied after
        st = ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
        assert st.ooc_devices == 2
    assert np.array_equal(C.astype(np.float64), og.gemm(A, B))


def test_single_group_all_tail():
    """n = 4, f = 4: pmm_run streams its inputs, so its groups are {0}, {1},
    {2, 3} (two single pivots first, runtime.cu setup); the whole k-loop is the
    tail and its first group overwrites C."""
    N, b = 512, 128
    A = synth.rect(3, N, 0, 0, N, N)
    B = synth.rect(4, N, 0, 0, N, N)
    C = np.full((N, N), np.nan, np.float32)
    with pkg.Context.local([0]) as ctx:
        ctx.set_option("e2e_tail", 16)
        st = ctx.run(A, B, C, N, b, [(0, 0, 0, 4, 4)], pkg.FPM_F32)
        assert st.updates == 3
    assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


def test_compute_into_pinned_windows():
    """pmm_compute_into into a pinned host matrix, twice on the same context,
    FP32 (tail) and FP64 (copied after the loop)."""
    N, b = 2048, 128
    n = N // b
    rects = pkg.colpart_arrange(n, [160, 96])
    for dt, tol in ((pkg.FPM_F32, 1e-5), (pkg.FPM_F64, 1e-12)):
        npdt = np.float32 if dt == pkg.FPM_F32 else np.float64
        tdt = torch.float32 if dt == pkg.FPM_F32 else torch.float64
        A = synth.rect(5, N, 0, 0, N, N, synth.DIST_PM1, npdt)
        B = synth.rect(6, N, 0, 0, N, N, synth.DIST_PM1, npdt)
        ref = og.gemm(A, B)
        with pkg.Context.local([0, 0]) as ctx:
            ctx.setup(N, b, rects, dt)
            ctx.fill_synthetic(5, 6)
            for _ in range(2):
                full = torch.full((N, N), float("nan"), dtype=tdt).pin_memory()
                st = ctx.compute_into(full, N)
                assert st.t_compute_s > 0
                assert og.rel_fro(full.numpy(), ref) <= tol


def test_nccl_single_rank_tail():
    N, b = 1024, 128
    A = synth.rect(7, N, 0, 0, N, N)
    B = synth.rect(8, N, 0, 0, N, N)
    C = np.full((N, N), np.nan, np.float32)
    with pkg.Context.nccl(0, 1, 0, pkg.Context.nccl_unique_id()) as ctx:
        ctx.set_option("e2e_tail", 2)
        ctx.run(A, B, C, N, b, [(0, 0, 0, N // b, N // b)], pkg.FPM_F32)
    assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


def test_e2e_tail_option_errors():
    with pkg.Context.local([0]) as ctx:
        for bad in (-2, 17):
            with pytest.raises(pkg.FpmError):
                ctx.set_option("e2e_tail", bad)


@pytest.mark.parametrize("stream", [1, 0])
@pytest.mark.parametrize("mode", ["run", "compute_into"])
def test_all_tail_repeated_calls(stream, mode):
    """The whole k-loop in the tail (e2e_tail >= the number of groups), called
    repeatedly on one context: the tail's first update must overwrite C_i, not
    add to the previous call's result (the streamed tail once hard-wired
    accumulation, which a fresh context's zeroed C hid)."""
    N, b = 2304, 96   # pmm_run groups {0}, {1}, 8, 8, 6: five groups, all in the tail
    n = N // b
    rects = pkg.colpart_arrange(n, [n * n])
    A = synth.rect(7, N, 0, 0, N, N)
    B = synth.rect(8, N, 0, 0, N, N)
    ref = og.gemm(A, B)
    with pkg.Context.local([0]) as ctx:
        ctx.set_option("e2e_tail", 16)
        ctx.set_option("tail_stream", stream)
        for _ in range(3):
            C = np.full((N, N), np.nan, np.float32)
            if mode == "run":
                ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
            else:
                ctx.setup(N, b, rects, pkg.FPM_F32)
                ctx.upload(A, B, N, 0, 0)
                ctx.compute_into(C, N, 0, 0)
            assert og.rel_fro(C, ref) <= 1e-5


@pytest.mark.parametrize("tail", [-1, 1, 3, 16])
@pytest.mark.parametrize("N,b", [(4096, 256), (2304, 96)])
def test_band_streamed_tail_matches_fused_tail(tail, N, b):
    """pmm_run on one device (option "tail_stream"): the tail's B rows are
    uploaded first and its A rows band by band, each band staged and updated as
    it lands.  Same operand, scales and sums as the fused tail: C bit-identical
    to tail_stream = 0, and within the FP32 tolerance of the oracle (integers:
    exact)."""
    n = N // b
    rects = pkg.colpart_arrange(n, [n * n])
    for dist in (synth.DIST_PM1, synth.DIST_INT):
        A = synth.rect(5, N, 0, 0, N, N, dist)
        B = synth.rect(6, N, 0, 0, N, N, dist)
        out = []
        for stream in (0, 1):
            C = np.full((N, N), np.nan, np.float32)
            with pkg.Context.local([0]) as ctx:
                # auto (-1): at these host-link-bound sizes the band-streamed
                # tail takes the whole k-loop (runtime.cu tail_groups), so the
                # fused tail it must match is the whole loop too
                ctx.set_option("e2e_tail", 16 if (tail == -1 and stream == 0) else tail)
                ctx.set_option("tail_stream", stream)
                ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
            out.append(C)
        assert np.array_equal(out[0], out[1])
        ref = og.gemm(A, B)
        if dist == synth.DIST_INT:
            assert np.array_equal(out[1].astype(np.float64), ref)
        else:
            assert og.rel_fro(out[1], ref) <= 1e-5


@pytest.mark.parametrize("tail", [-1, 1, 3])
@pytest.mark.parametrize("mode", ["compute_into", "run"])
def test_fused_staging_with_tail_bit_identical(tail, mode):
    """In-kernel staging (forced: option fused_staging = 2) up to the download
    tail: the last non-tail update stages nothing, the tail groups take the
    standalone staging (fused tail operand / band-streamed tail); C
    bit-identical to fused_staging = 0, integers bit-exact vs the oracle."""
    N, b = 4096, 256
    n = N // b
    rects = pkg.colpart_arrange(n, [n * n])
    A = synth.rect(21, N, 0, 0, N, N, synth.DIST_INT)
    B = synth.rect(22, N, 0, 0, N, N, synth.DIST_INT)
    out = []
    for fs in (2, 0):
        C = np.full((N, N), np.nan, np.float32)
        with pkg.Context.local([0]) as ctx:
            ctx.set_option("fused_staging", fs)
            ctx.set_option("e2e_tail", tail)
            if mode == "run":
                ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
            else:
                ctx.setup(N, b, rects, pkg.FPM_F32)
                ctx.upload(A, B, N)
                ctx.compute_into(C, N)
        out.append(C)
    assert np.array_equal(out[0], out[1])
    assert np.array_equal(out[0].astype(np.float64), og.gemm(A, B))
