"""End-to-end parity of the hot path on the GPU, through the C ABI:
fpm_partition -> colpart_arrange -> pmm_run (pivot exchange + staging + rank-b
updates) vs the oracle GEMM; fpm_sample procedure checks; full-size sampled
parity at the bench configuration."""
import numpy as np
import pytest

import synth
from oracle import fpm as ofpm
from oracle import gemm as og

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402


@pytest.fixture(autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    yield


def _models(seed, p):
    return synth.random_models(np.random.default_rng(seed), p, monotone_time=True, max_m=12)


def _run(ctx, N, b, rects, dt, dist=synth.DIST_PM1, seeds=(1, 2)):
    npdt = np.float32 if dt == pkg.FPM_F32 else np.float64
    A = synth.rect(seeds[0], N, 0, 0, N, N, dist, npdt)
    B = synth.rect(seeds[1], N, 0, 0, N, N, dist, npdt)
    C = np.full((N, N), np.nan, dtype=npdt)
    st = ctx.run(A, B, C, N, b, rects, dt)
    return A, B, C, st


@pytest.mark.parametrize("dt,tol", [(pkg.FPM_F32, 1e-5), (pkg.FPM_F64, 1e-12)])
@pytest.mark.parametrize("N,b", [(512, 64), (1024, 128), (768, 256)])
def test_p1(dt, tol, N, b):
    with pkg.Context.local([0]) as ctx:
        A, B, C, st = _run(ctx, N, b, [(0, 0, 0, N // b, N // b)], dt)
        assert og.rel_fro(C, og.gemm(A, B)) <= tol
        assert st.iters == N // b and st.t_compute_s > 0 and st.kernel_launches > 0


@pytest.mark.parametrize("p", [2, 3, 4, 5])
@pytest.mark.parametrize("dt", [pkg.FPM_F32, pkg.FPM_F64])
def test_local_multi_device_parity(p, dt):
    """p emulated devices on one GPU: FPM partition, arrangement, pivot exchange."""
    N, b = 768, 64
    n = N // b
    models = _models(100 + p, p)
    d = pkg.fpm_partition(n * n, models)
    assert d == ofpm.partition(n * n, models)
    rects = pkg.colpart_arrange(n, d)
    assert rects == ofpm.arrange(n, d)
    with pkg.Context.local([0] * p) as ctx:
        A, B, C, st = _run(ctx, N, b, rects, dt)
        tol = 1e-5 if dt == pkg.FPM_F32 else 1e-12
        assert og.rel_fro(C, og.gemm(A, B)) <= tol
        live = [i for i, r in enumerate(rects) if r[3] * r[4] > 0]
        assert all(st.per_dev_compute_s[i] > 0 for i in live)
        if len(live) > 1:
            assert st.comm_bytes > 0


@pytest.mark.parametrize("p", [1, 2, 4, 8])
def test_integer_inputs_bit_exact_and_p_invariant(p):
    N, b = 1024, 128
    n = N // b
    d = pkg.fpm_partition(n * n, [([1], [1.0 + i % 3]) for i in range(p)])
    rects = pkg.colpart_arrange(n, d)
    ref = None
    for dt in (pkg.FPM_F32, pkg.FPM_F64):
        with pkg.Context.local([0] * p) as ctx:
            A, B, C, _ = _run(ctx, N, b, rects, dt, dist=synth.DIST_INT, seeds=(11, 12))
        exact = og.gemm(A, B)
        assert np.array_equal(C.astype(np.float64), exact)
        ref = exact if ref is None else ref


@pytest.mark.parametrize("fuse", [1, 2, 3, 8])
def test_fused_pivot_groups(fuse):
    """f pivots per update (groups cut at every column / row boundary), local
    fused pulls, FP32: parity with the oracle, integer inputs bit-exact."""
    N, b = 1536, 64
    n = N // b
    rects = pkg.colpart_arrange(n, [250, 170, 96, 60])
    with pkg.Context.local([0] * 4) as ctx:
        ctx.set_option("fuse", fuse)
        A, B, C, st = _run(ctx, N, b, rects, pkg.FPM_F32)
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5
        assert st.updates >= -(-n // fuse)
        Ai, Bi, Ci, _ = _run(ctx, N, b, rects, pkg.FPM_F32, dist=synth.DIST_INT, seeds=(7, 8))
        assert np.array_equal(Ci.astype(np.float64), og.gemm(Ai, Bi))


def test_streamed_run_starts_with_single_pivots():
    """pmm_run (host-streamed inputs) groups {0}, {1}, {2..9}, {10..15} at
    n = 16, f = 8; pmm_compute on resident inputs {0..7}, {8..15}.  Same C
    within tolerance, integer inputs bit-exact on both."""
    N, b = 2048, 128
    n = N // b
    rects = [(0, 0, 0, n, n)]
    with pkg.Context.local([0]) as ctx:
        ctx.set_option("fuse", 8)
        A, B, C, st = _run(ctx, N, b, rects, pkg.FPM_F32)
        assert st.updates == 4
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5
        ctx.upload(A, B, N)
        assert ctx.compute().updates == 2
        Cr = np.full((N, N), np.nan, np.float32)
        ctx.download(Cr, N)
        assert og.rel_fro(Cr, og.gemm(A, B)) <= 1e-5
        Ai, Bi, Ci, st = _run(ctx, N, b, rects, pkg.FPM_F32, dist=synth.DIST_INT, seeds=(7, 8))
        assert np.array_equal(Ci.astype(np.float64), og.gemm(Ai, Bi)) and st.updates == 4


@pytest.mark.parametrize("seed", [3, 4])
def test_run_on_fpm_arrangement(seed):
    """colpart_arrange_fpm rectangles (integers chosen on the models, Q25):
    same exchange and update path, parity with the oracle."""
    N, b = 1536, 64
    n = N // b
    models = _models(seed, 5)
    d = pkg.fpm_partition(n * n, models)
    rects = pkg.colpart_arrange_fpm(n, d, models)
    assert rects == ofpm.arrange_fpm(n, d, models)
    with pkg.Context.local([0] * 5) as ctx:
        A, B, C, st = _run(ctx, N, b, rects, pkg.FPM_F32)
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5
        A, B, C, st = _run(ctx, N, b, rects, pkg.FPM_F64)
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-12


def test_kernel_launch_count():
    """pmm_stats.kernel_launches counts every library kernel of the k-loop: per
    update group one A split, three B-row kernels (maxima, split, scales) for
    F16X3 or one for TF32X3, and the update; with in-kernel staging (F16X3
    default) only the first group's staging kernels run, the later groups are
    staged by the previous update's staging warp."""
    N, b = 2048, 128
    n = N // b
    with pkg.Context.local([0]) as ctx:
        ctx.set_option("fuse", 8)
        ctx.set_option("fused_staging", 2)
        ctx.setup(N, b, [(0, 0, 0, n, n)], pkg.FPM_F32)
        ctx.fill_synthetic(1, 2)
        for graph in (0, 1):
            ctx.set_option("graph", graph)
            st = ctx.compute()
            assert st.updates == 2 and st.kernel_launches == (1 + 3) + 2
        ctx.set_option("fused_staging", 0)
        for graph in (0, 1):
            ctx.set_option("graph", graph)
            st = ctx.compute()
            assert st.updates == 2 and st.kernel_launches == 2 * (1 + 3 + 1)
        ctx.set_option("f32_scheme", pkg.SCHEME_TF32X3)
        ctx.setup(N, b, [(0, 0, 0, n, n)], pkg.FPM_F32)
        ctx.fill_synthetic(1, 2)
        assert ctx.compute().kernel_launches == 2 * (1 + 1 + 1)


def test_single_iteration_b_equals_n():
    """n = 1: one pivot, one update that overwrites C."""
    N = b = 512
    with pkg.Context.local([0]) as ctx:
        for dt, tol in ((pkg.FPM_F32, 1e-5), (pkg.FPM_F64, 1e-12)):
            A, B, C, st = _run(ctx, N, b, [(0, 0, 0, 1, 1)], dt)
            assert og.rel_fro(C, og.gemm(A, B)) <= tol and st.iters == 1 and st.updates == 1


def test_sixteen_devices_and_ragged_tiles():
    """p = 16 (the ABI maximum) emulated devices; rectangle sides that are not
    multiples of the 256-row tile (b = 96)."""
    N, b = 96 * 20, 96
    n = N // b
    models = _models(77, 16)
    d = pkg.fpm_partition(n * n, models)
    assert d == ofpm.partition(n * n, models)
    rects = pkg.colpart_arrange(n, d)
    with pkg.Context.local([0] * 16) as ctx:
        A, B, C, st = _run(ctx, N, b, rects, pkg.FPM_F32, dist=synth.DIST_INT, seeds=(3, 4))
        assert np.array_equal(C.astype(np.float64), og.gemm(A, B))


def test_tf32x3_scheme_and_cta_group1():
    N, b = 1024, 128
    rects = pkg.colpart_arrange(N // b, [32, 32])
    for scheme, cg in [(pkg.SCHEME_TF32X3, 2), (pkg.SCHEME_F16X3, 1), (pkg.SCHEME_TF32X3, 1)]:
        with pkg.Context.local([0, 0]) as ctx:
            ctx.set_option("f32_scheme", scheme)
            ctx.set_option("cta_group", cg)
            A, B, C, _ = _run(ctx, N, b, rects, pkg.FPM_F32)
            assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


def test_zero_area_device_and_sm_caps():
    N, b = 512, 64
    n = N // b
    d = [n * n - 5, 5, 0]
    rects = pkg.colpart_arrange(n, d)
    with pkg.Context.local([0, 0, 0], sm_caps=[64, 16, 8]) as ctx:
        A, B, C, st = _run(ctx, N, b, rects, pkg.FPM_F32)
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


def test_nccl_mode_single_rank():
    """The NCCL context (dlopen'ed libnccl, world communicator, column split) on
    one rank: exercises the multi-process code path end to end on one GPU."""
    nid = pkg.Context.nccl_unique_id()
    with pkg.Context.nccl(0, 1, 0, nid) as ctx:
        A, B, C, st = _run(ctx, 512, 64, [(0, 0, 0, 8, 8)], pkg.FPM_F32)
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


def test_run_streams_host_windows():
    """pmm_run with a host window that is only one device's rectangle (the
    multi-process usage) and with pinned host memory."""
    N, b = 1024, 128
    n = N // b
    rects = pkg.colpart_arrange(n, [40, 24])
    A = synth.rect(1, N, 0, 0, N, N)
    B = synth.rect(2, N, 0, 0, N, N)
    hA = torch.from_numpy(A).pin_memory()
    hB = torch.from_numpy(B).pin_memory()
    hC = torch.full((N, N), float("nan")).pin_memory()
    with pkg.Context.local([0, 0]) as ctx:
        st = ctx.run(hA, hB, hC, N, b, rects, pkg.FPM_F32)
        assert st.t_upload_s > 0 and st.t_download_s > 0
    assert og.rel_fro(hC.numpy(), og.gemm(A, B)) <= 1e-5
    # host arrays with a leading dimension larger than N (padded rows)
    pad = 24
    Ap = np.full((N, N + pad), 5.0, np.float32)
    Bp = np.full((N, N + pad), 5.0, np.float32)
    Ap[:, :N], Bp[:, :N] = A, B
    Cp = np.full((N, N + pad), np.nan, dtype=np.float32)
    with pkg.Context.local([0]) as ctx:
        ctx.run(Ap, Bp, Cp, N, b, [(0, 0, 0, n, n)], pkg.FPM_F32, ld=N + pad)
    assert og.rel_fro(Cp[:, :N], og.gemm(A, B)) <= 1e-5
    assert np.all(np.isnan(Cp[:, N:]))


def test_invalid_arguments_fail_loudly():
    with pkg.Context.local([0]) as ctx:
        with pytest.raises(pkg.FpmError):
            ctx.setup(500, 64, [(0, 0, 0, 7, 7)])        # b does not divide N
        with pytest.raises(pkg.FpmError):
            ctx.setup(512, 64, [(0, 0, 0, 8, 7)])        # does not tile
        with pytest.raises(pkg.FpmError):
            ctx.compute()                                 # no problem set
    with pytest.raises(pkg.FpmError):
        pkg.Context.local([0], sm_caps=[13])              # odd: CTA pairs need an even cap


def test_fpm_sample_procedure():
    """Speed points are positive, meet the CI stop rule or the repetition cap (P:10 (iii))."""
    with pkg.Context.local([0]) as ctx:
        sizes = [1, 4, 16, 64]
        sp, ci, reps = ctx.sample(0, 256, sizes, pkg.FPM_F32)
        assert all(s > 0 for s in sp)
        assert all(5 <= r <= 50 for r in reps)
        assert all(c <= 0.025 or r == 50 for c, r in zip(ci, reps))
        sp64, _, _ = ctx.sample(0, 64, [1, 4, 9], pkg.FPM_F64)
        assert all(s > 0 for s in sp64)
        with pytest.raises(pkg.FpmError):
            ctx.sample(0, 256, [3])                        # not a perfect square


@pytest.mark.parametrize("cap", [0, 64])
def test_fpm_sample_through_fused_staging(cap):
    """Where the k-loop stages the next group inside the update (sizes from
    about 5000^2 on a device alone on its GPU), fpm_sample times that path:
    each timed update stages the next run's operands in-kernel.  At such
    sizes the sampled speeds are positive and converge, in-kernel sampling is
    no slower than the standalone split + update it replaces (option
    fused_staging = 0), and the same context's run afterwards is correct."""
    b, ms = 512, [4, 12, 16]
    sizes = [m * m for m in ms]
    caps = [cap] if cap else None
    with pkg.Context.local([0], sm_caps=caps) as ctx:
        sp, ci, reps = ctx.sample(0, b, sizes, pkg.FPM_F32)
        assert all(s > 0 for s in sp) and all(5 <= r <= 50 for r in reps)
        ctx.set_option("fused_staging", 0)
        sp0, _, _ = ctx.sample(0, b, sizes, pkg.FPM_F32)
        ctx.set_option("fused_staging", 1)
        assert sp[2] >= 0.95 * sp0[2], (sp, sp0)   # 8192^2: in-kernel staging applies
        N = 2048
        n = N // b
        A, B = synth.rect(31, N, 0, 0, N, N), synth.rect(32, N, 0, 0, N, N)
        C = np.full((N, N), np.nan, np.float32)
        ctx.run(A, B, C, N, b, [(0, 0, 0, n, n)], pkg.FPM_F32)
    assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


def test_fpm_sample_all_devices_concurrently():
    """dev = -1: every device sampled at once (P:10 (ii)); a device capped to
    fewer SMs must come out slower at a size that fills the GPU."""
    with pkg.Context.local([0, 0], sm_caps=[96, 32]) as ctx:
        sp, ci, reps = ctx.sample(-1, 512, [64, 256], pkg.FPM_F32)
        assert len(sp) == 2 and all(len(r) == 2 for r in sp)
        assert all(s > 0 for row in sp for s in row)
        assert sp[0][1] > 1.5 * sp[1][1]


def test_config1_fp64_two_capped_devices():
    """BASELINE config 1: N=512, b=64, FP64, two emulated devices in DISJOINT
    green-context SM partitions of the GPU, caps {100, 48} (reading Q13): FPMs
    from 8 sample sizes -> partition (bit-exact vs the oracle) -> arrangement ->
    multiply (within 1e-12 of the oracle)."""
    from oracle import fpm as ofpm
    N, b = 512, 64
    n = N // b
    sizes = [m * m for m in range(1, 9)]
    with pkg.Context.local([0, 0], sm_caps=[100, 48]) as ctx:
        ctx.set_option("sm_partition", 1)
        models = []
        for dev in range(2):
            sp, _, _ = ctx.sample(dev, b, sizes, pkg.FPM_F64)
            models.append((sizes, sp))
        d = pkg.fpm_partition(n * n, models)
        assert sum(d) == n * n and d == ofpm.partition(n * n, models)
        rects = pkg.colpart_arrange(n, d)
        assert rects == ofpm.arrange(n, d)
        A, B, C, _ = _run(ctx, N, b, rects, pkg.FPM_F64, seeds=(1, 2))
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-12


@pytest.mark.parametrize("N,b", [(16384, 512), (49152, 1024)])
def test_full_size_sampled_parity(N, b):
    """Bench configurations (c3 at p=1, c5 at p=1): synthetic inputs generated on
    the device by the shared counter-based generator, sampled blocks of C
    (corners, interior, ragged tile edges) vs the oracle on the same entries."""
    free, _ = torch.cuda.mem_get_info(0)
    if free < 3.3 * 3 * N * N * 4:
        pytest.skip("not enough device memory")
    n = N // b
    with pkg.Context.local([0]) as ctx:
        ctx.setup(N, b, [(0, 0, 0, n, n)], pkg.FPM_F32)
        ctx.fill_synthetic(1, 2, pkg.FPM_DIST_PM1)
        st = ctx.compute(zero_c=True)
        assert st.t_compute_s > 0
        rng = np.random.default_rng(N)
        blocks = [(0, 0), (N - 16, N - 64), (0, N - 64), (N - 16, 0)]
        blocks += [(int(r), int(c)) for r, c in zip(rng.integers(0, N - 16, 4), rng.integers(0, N - 64, 4))]
        B_cols = {}
        for (r0, c0) in blocks:
            got = ctx.download_block(r0, c0, 16, 64)
            A_rows = synth.rect(1, N, r0, 0, 16, N)
            if c0 not in B_cols:
                B_cols[c0] = synth.rect(2, N, 0, c0, N, 64)
            ref = og.gemm(A_rows, B_cols[c0])
            assert og.rel_fro(got, ref) <= 1e-5, (r0, c0, og.rel_fro(got, ref))


@pytest.mark.parametrize("sm_partition", [0, 1])
def test_c4_full_size_sampled_parity(sm_partition):
    """Config 4 at full size (N = 32768, b = 512, 8 devices with the SM caps of the
    heterogeneity study, grid caps or green partitions), an FPM partition of
    synthetic speed functions and the column arrangement: sampled blocks of C
    in every device's rectangle (corners and an interior block) vs the oracle."""
    N, b = 32768, 512
    free, _ = torch.cuda.mem_get_info(0)
    if free < 3.3 * 3 * N * N * 4:
        pytest.skip("not enough device memory")
    n = N // b
    caps = [30, 26, 24, 20, 16, 14, 10, 6]
    sizes = [1, 4, 16, 64, 256, 1024, 4096]
    models = [(sizes, [c * (1.0 - 0.5 / (1 + x / 16.0)) for x in sizes]) for c in caps]
    d = pkg.fpm_partition(n * n, models)
    rects = pkg.colpart_arrange(n, d)
    try:
        ctx = pkg.Context.local([0] * 8, sm_caps=caps)
    except pkg.FpmError:
        pytest.skip("SM caps not available")
    with ctx:
        ctx.set_option("sm_partition", sm_partition)
        try:
            ctx.setup(N, b, rects, pkg.FPM_F32)
        except pkg.FpmError as ex:
            if sm_partition:
                pytest.skip(f"green partitions unavailable: {ex}")
            raise
        ctx.fill_synthetic(1, 2, pkg.FPM_DIST_PM1)
        st = ctx.compute(zero_c=True)
        assert st.t_compute_s > 0
        B_cols = {}
        for (col, r_0, c_0, h, w) in rects:
            if h * w == 0:
                continue
            R0, C0, H, W = r_0 * b, c_0 * b, h * b, w * b
            for (r0, c0) in [(R0, C0), (R0 + H - 16, C0 + W - 64), (R0 + H // 2, C0 + W // 2)]:
                got = ctx.download_block(r0, c0, 16, 64)
                A_rows = synth.rect(1, N, r0, 0, 16, N)
                if c0 not in B_cols:
                    B_cols[c0] = synth.rect(2, N, 0, c0, N, 64)
                ref = og.gemm(A_rows, B_cols[c0])
                assert og.rel_fro(got, ref) <= 1e-5, (r0, c0, og.rel_fro(got, ref))


def test_sample_rects_gpu():
    """fpm_sample_rects (reading Q26): a square rectangle times like fpm_sample's
    square size (within the sampling noise), a near-square rectangle of the
    same area likewise, and dev = -1 samples every device on its own
    shape at once (2 devices: the 96-SM device's larger rectangle)."""
    with pkg.Context.local([0, 0], sm_caps=[96, 48]) as ctx:
        sq, _, _ = ctx.sample(0, 512, [64], pkg.FPM_F32)
        r, ci, reps = ctx.sample_rects(0, 512, [(8, 8), (4, 16)], pkg.FPM_F32)
        assert all(v > 0 for v in r) and all(n >= 5 for n in reps)
        assert abs(r[0] / sq[0] - 1) < 0.15
        assert abs(r[1] / r[0] - 1) < 0.2
        sp, _, _ = ctx.sample_rects(-1, 512, [[(12, 12)], [(6, 6)]], pkg.FPM_F32)
        assert len(sp) == 2 and sp[0][0] > sp[1][0] > 0
        with pytest.raises(pkg.FpmError):
            ctx.sample_rects(0, 512, [(0, 4)], pkg.FPM_F32)


def test_per_device_span_stats():
    """pmm_stats.per_dev_span_s: every live device's k-loop span is positive, at
    most the k-loop time (its maximum), at least its summed update time; a
    zero-area device reports 0."""
    N, b = 2048, 256
    n = N // b
    rects = pkg.colpart_arrange(n, [40, 24, 0])
    with pkg.Context.local([0, 0, 0]) as ctx:
        ctx.setup(N, b, rects, pkg.FPM_F32)
        ctx.fill_synthetic(1, 2, pkg.FPM_DIST_PM1)
        st = ctx.compute()
        for i in range(2):
            assert 0 < st.per_dev_update_s[i] <= st.per_dev_span_s[i] * 1.001
            assert st.per_dev_span_s[i] <= st.t_compute_s * 1.001
        assert max(st.per_dev_span_s[:2]) == pytest.approx(st.t_compute_s, rel=1e-6)
        assert st.per_dev_span_s[2] == 0.0


@pytest.mark.parametrize("graph", [1, 0])
def test_group_times_timeline(graph):
    """pmm_group_times: one (staging start, end, update start, end) record per
    update group; each interval ordered, a group's update starts after its own
    staging ended, updates follow each other on the compute stream, and their
    summed length is the per-device update time of pmm_stats."""
    N, b = 2048, 256
    n = N // b
    rects = pkg.colpart_arrange(n, [40, 24])
    with pkg.Context.local([0, 0]) as ctx:
        ctx.set_option("graph", graph)
        ctx.setup(N, b, rects, pkg.FPM_F32)
        ctx.fill_synthetic(1, 2, pkg.FPM_DIST_PM1)
        ctx.compute()
        st = ctx.compute()
        for dev in range(2):
            tl = ctx.group_times(dev)
            assert len(tl) == st.updates
            prev_end = 0.0
            for p0, p1, u0, u1 in tl:
                assert 0.0 <= p0 <= p1 <= u0 <= u1 <= st.t_compute_s * 1.001
                assert u0 >= prev_end * 0.999999
                prev_end = u1
            assert sum(u1 - u0 for _, _, u0, u1 in tl) == pytest.approx(st.per_dev_update_s[dev], rel=1e-4)
        with pytest.raises(pkg.FpmError):
            ctx.group_times(5)


@pytest.mark.parametrize("N,b,fuse", [(3072, 256, 0), (2880, 96, 3), (4096, 512, 1), (1024, 128, 2)])
@pytest.mark.parametrize("graph", [1, 0])
def test_fused_staging_bit_identical(N, b, fuse, graph):
    """Option fused_staging (default on): update g's staging warp stages group
    g + 1 (kernels.hpp StageJob) instead of the standalone split kernels between
    the updates.  Same arithmetic (split_math.cuh), so C is bit-identical with
    the option off, eager or graph-replayed, with ragged column chunks (W not a
    multiple of 128), one / several pivots per update, and repeated computes
    (the grid-barrier counters re-arm); and C matches the oracle."""
    n = N // b
    rects = pkg.colpart_arrange(n, [n * n])
    out = []
    for fs in (2, 0):   # 2: in-kernel staging at these (small) sizes too
        with pkg.Context.local([0]) as ctx:
            ctx.set_option("graph", graph)
            ctx.set_option("fuse", fuse)
            ctx.set_option("fused_staging", fs)
            ctx.setup(N, b, rects, pkg.FPM_F32)
            ctx.fill_synthetic(1, 2, pkg.FPM_DIST_PM1)
            for _ in range(3):
                st = ctx.compute()
            C = np.empty((N, N), np.float32)
            ctx.download(C, N)
            out.append((C, st.kernel_launches, ctx.group_times(0)))
    assert np.array_equal(out[0][0], out[1][0])
    assert out[0][1] < out[1][1]          # no standalone staging kernels after the first group
    tl = out[0][2]
    assert all(p1 - p0 < 1e-4 for p0, p1, _, _ in tl[1:])   # staged inside the updates (no staging interval)
    ref = og.gemm(synth.rect(1, N, 0, 0, N, N), synth.rect(2, N, 0, 0, N, N))
    assert og.rel_fro(out[0][0], ref) <= 1e-5


@pytest.mark.parametrize("N,b,dist", [(4096, 512, synth.DIST_INT), (3072, 256, synth.DIST_PM1)])
@pytest.mark.parametrize("tail_stream", [1, 0])
def test_fused_staging_streamed_run(N, b, dist, tail_stream):
    """pmm_run (host panels streamed in under the k-loop) with in-kernel
    staging: the staging warp waits for the upload-progress flag of the next
    group's panels; C bit-identical to fused_staging = 0 over repeated runs
    (the flag epochs advance), integer inputs bit-exact vs the oracle."""
    n = N // b
    rects = pkg.colpart_arrange(n, [n * n])
    A = synth.rect(1, N, 0, 0, N, N, dist)
    B = synth.rect(2, N, 0, 0, N, N, dist)
    out = []
    for fs in (2, 0):
        with pkg.Context.local([0]) as ctx:
            ctx.set_option("fused_staging", fs)
            ctx.set_option("tail_stream", tail_stream)
            for _ in range(2):
                C = np.full((N, N), np.nan, dtype=np.float32)
                ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
            out.append(C)
    assert np.array_equal(out[0], out[1])
    ref = og.gemm(A, B)
    if dist == synth.DIST_INT:
        assert np.array_equal(out[0].astype(np.float64), ref)
    else:
        assert og.rel_fro(out[0], ref) <= 1e-5


@pytest.mark.parametrize("graph", [1, 0])
def test_shared_b_operand_bit_identical(graph):
    """Option share_b (default on): column members on the B owner's GPU read its
    staged B operand.  The operand is the same bytes either way (same rows,
    same column maxima), so C is bit-identical to share_b = 0, with the k-loop
    replayed as a graph or issued eagerly, and repeated computes agree."""
    N, b = 3072, 256
    n = N // b
    rects = pkg.colpart_arrange(n, [40, 36, 30, 20, 18])
    assert len({r[0] for r in rects}) < 5     # some columns hold several devices
    out = []
    for share in (1, 0):
        with pkg.Context.local([0] * 5) as ctx:
            ctx.set_option("graph", graph)
            ctx.set_option("share_b", share)
            ctx.setup(N, b, rects, pkg.FPM_F32)
            ctx.fill_synthetic(1, 2, pkg.FPM_DIST_PM1)
            ctx.compute()
            ctx.compute()
            C = np.empty((N, N), np.float32)
            ctx.download(C, N)
            out.append(C)
    assert np.array_equal(out[0], out[1])
    ref = og.gemm(synth.rect(1, N, 0, 0, N, N), synth.rect(2, N, 0, 0, N, N))
    assert og.rel_fro(out[0], ref) <= 1e-5
