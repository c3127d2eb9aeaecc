"""Host-CPU devices (§III, §V: sockets of c cores running
the GEMM kernel simultaneously, partitioned together with the GPUs; SURVEY
§8(f) NEXT-3).  These run WITHOUT a GPU: the CPU device's GEMM
(fpm_k_cpu_gemm) and contexts made only of CPU devices, through the C ABI,
against the oracle (plain triple loop, FP64 accumulation).  Mixed CPU + GPU
contexts are in tests/test_gpu_cpu_devices.py."""
import numpy as np
import pytest

import synth
from oracle import fpm as ofpm
from oracle import gemm as og

import paper_conf_cluster_zhongrl12_b200 as pkg

CPU = pkg.FPM_CPU_DEVICE
NCORES = len(pkg.cpu_cores())


def test_isa_and_cores():
    assert pkg.cpu_isa() in ("avx512", "avx2", "generic")
    cores = pkg.cpu_cores()
    assert len(cores) >= 1 and cores == sorted(cores)


@pytest.mark.parametrize("dt,tol", [(np.float32, 1e-5), (np.float64, 1e-12)])
@pytest.mark.parametrize("M,N,K", [(1, 1, 1), (5, 7, 3), (37, 45, 29), (100, 257, 300), (129, 65, 513)])
@pytest.mark.parametrize("threads", [1, 3])
def test_cpu_gemm_vs_oracle(dt, tol, M, N, K, threads):
    rng = np.random.default_rng(M * 1000 + N + K)
    A = rng.uniform(-1, 1, (M, K)).astype(dt)
    B = rng.uniform(-1, 1, (K, N)).astype(dt)
    C = np.full((M, N), np.nan, dt)
    pkg.k_cpu_gemm(A, B, C, threads=threads)
    assert og.rel_fro(C, og.gemm(A, B)) <= tol


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_cpu_gemm_accumulate_and_strides(dt):
    """C (+)= A B with leading dimensions larger than the shapes (a window of a
    bigger matrix), accumulate into an existing C."""
    rng = np.random.default_rng(3)
    big_A = rng.uniform(-1, 1, (90, 130)).astype(dt)
    big_B = rng.uniform(-1, 1, (130, 170)).astype(dt)
    big_C = rng.uniform(-1, 1, (95, 180)).astype(dt)
    A, B, C = big_A[5:75, 10:110], big_B[10:110, 20:150], big_C[3:73, 40:170]
    ref = og.gemm(np.ascontiguousarray(A), np.ascontiguousarray(B)) + C.astype(np.float64)
    outside = big_C.copy()
    pkg.k_cpu_gemm(A, B, C, accumulate=True, threads=2)
    tol = 1e-5 if dt == np.float32 else 1e-12
    assert og.rel_fro(C, ref) <= tol
    mask = np.ones(big_C.shape, bool)
    mask[3:73, 40:170] = False
    np.testing.assert_array_equal(big_C[mask], outside[mask])   # nothing outside the window written


@pytest.mark.parametrize("seg", [1, 7, 32, 64])
def test_cpu_gemm_k_segments(seg):
    """A read in K-segments (a device's block-column panels: A(i, k) at
    (k / seg) * seg_stride + i * lda + k % seg) equals the same matrix stored plainly."""
    M, K, N = 50, 128, 40
    rng = np.random.default_rng(seg)
    A = rng.integers(-8, 9, (M, K)).astype(np.float32)
    B = rng.integers(-8, 9, (K, N)).astype(np.float32)
    nseg = -(-K // seg)
    panels = np.zeros((nseg, M, seg), np.float32)
    for j in range(nseg):
        w = min(seg, K - j * seg)
        panels[j, :, :w] = A[:, j * seg:j * seg + w]
    C = np.empty((M, N), np.float32)
    pkg.k_cpu_gemm(panels, B, C, M=M, N=N, K=K, lda=seg, seg=seg, seg_stride=M * seg, threads=2)
    np.testing.assert_array_equal(C, (A.astype(np.int64) @ B.astype(np.int64)).astype(np.float32))


def test_cpu_gemm_integers_bit_exact():
    """Integers in [-8, 8], K = 1000: every partial sum < 2^24, so FP32 is exact."""
    A = synth.rect(5, 1000, 0, 0, 300, 1000, synth.DIST_INT)
    B = synth.rect(6, 1000, 0, 0, 1000, 200, synth.DIST_INT)
    C = np.empty((300, 200), np.float32)
    pkg.k_cpu_gemm(A, B, C, threads=min(4, NCORES))
    np.testing.assert_array_equal(C, og.gemm(A, B).astype(np.float32))


def test_cpu_gemm_rejects_bad_args():
    A = np.zeros((4, 4), np.float32)
    with pytest.raises(pkg.FpmError):
        pkg.k_cpu_gemm(A, A, A, threads=0)
    with pytest.raises(pkg.FpmError):
        pkg.k_cpu_gemm(A, A, A, threads=NCORES + 1, pin=True)


def _cores_each(p):
    c = max(1, NCORES // p)
    if c * p > NCORES:
        pytest.skip("not enough host cores")
    return [c] * p


@pytest.mark.parametrize("dt,tol", [(pkg.FPM_F32, 1e-5), (pkg.FPM_F64, 1e-12)])
@pytest.mark.parametrize("d", [[64], [40, 24], [30, 20, 10, 4]])
def test_cpu_only_context_run_parity(dt, tol, d):
    """fpm arrangement -> pmm_run on a context of CPU devices only (P:15 on the
    paper's CPUs-only configuration, Table II column 2): C vs the oracle."""
    N, b = 512, 64
    n = N // b
    rects = pkg.colpart_arrange(n, d)
    npdt = np.float32 if dt == pkg.FPM_F32 else np.float64
    A = synth.rect(1, N, 0, 0, N, N).astype(npdt)
    B = synth.rect(2, N, 0, 0, N, N).astype(npdt)
    C = np.full((N, N), np.nan, npdt)
    with pkg.Context.local([CPU] * len(d), sm_caps=_cores_each(len(d))) as ctx:
        st = ctx.run(A, B, C, N, b, rects, dt)
    assert og.rel_fro(C, og.gemm(A, B)) <= tol
    live = [i for i, r in enumerate(rects) if r[3] * r[4] > 0]
    assert all(st.per_dev_compute_s[i] > 0 for i in live)
    assert st.t_compute_s >= max(st.per_dev_update_s[i] for i in live)
    # pivot bytes received: sum over devices and iterations of the pieces not held locally
    expect = 0
    for k in range(n):
        a_moves, b_moves = pkg.colpart_plan_step(n, rects, k)
        expect += sum((m[3] - m[2]) * b * b for m in a_moves if m[0] != m[1])
        expect += sum(rects[m[1]][4] * b * b for m in b_moves if m[0] != m[1])
    assert st.comm_bytes == expect * npdt().itemsize


def test_cpu_only_integers_exact_and_fill_synthetic():
    """Integer inputs, on-device (host) synthetic fill by the shared generator,
    sampled blocks bit-exact."""
    N, b = 640, 64
    n = N // b
    rects = pkg.colpart_arrange(n, [50, 30, 20])
    with pkg.Context.local([CPU] * 3, sm_caps=_cores_each(3)) as ctx:
        ctx.setup(N, b, rects, pkg.FPM_F32)
        ctx.fill_synthetic(11, 12, pkg.FPM_DIST_INT)
        ctx.compute()
        for (_, r0, c0, h, w) in rects:
            R0, C0 = r0 * b + 3, c0 * b + 5
            got = ctx.download_block(R0, C0, 8, 9)
            ref = og.gemm(synth.rect(11, N, R0, 0, 8, N, synth.DIST_INT), synth.rect(12, N, 0, C0, N, 9, synth.DIST_INT))
            np.testing.assert_array_equal(got, ref.astype(np.float32))


def test_cpu_device_fpm_sample_procedure():
    """fpm_sample on a CPU device: positive speeds, the Q8 stop rule (>= 5
    repetitions, CI <= 2.5 % or 50 repetitions), perfect squares only."""
    with pkg.Context.local([CPU], sm_caps=[min(2, NCORES)]) as ctx:
        sp, ci, reps = ctx.sample(0, 64, [1, 4, 16], pkg.FPM_F32)
        assert all(s > 0 for s in sp)
        assert all(5 <= r <= 50 for r in reps)
        assert all(c <= 0.025 or r == 50 for c, r in zip(ci, reps))
        with pytest.raises(pkg.FpmError):
            ctx.sample(0, 64, [2], pkg.FPM_F32)


def test_cpu_devices_synchronised_sampling():
    """fpm_sample(dev = -1) on CPU devices: all devices' windows in step (P:10
    (ii)); per-device lists of positive speeds under the Q8 stop rule, and
    fpm_sample_rects(-1) with a rectangle per device."""
    if NCORES < 2:
        pytest.skip("needs 2 host cores")
    with pkg.Context.local([CPU, CPU], sm_caps=[1, 1]) as ctx:
        sp, ci, reps = ctx.sample(-1, 64, [1, 4], pkg.FPM_F32)
        assert len(sp) == 2 and all(len(r) == 2 for r in sp)
        assert all(v > 0 for r in sp for v in r)
        assert all(5 <= n <= 50 for r in reps for n in r)
        assert all(c <= 0.025 or n == 50 for cr, rr in zip(ci, reps) for c, n in zip(cr, rr))
        sp2, _, _ = ctx.sample_rects(-1, 64, [[(2, 3)], [(1, 2)]], pkg.FPM_F32)
        assert len(sp2) == 2 and sp2[0][0] > 0 and sp2[1][0] > 0


def test_cpu_device_fpm_partition_end_to_end():
    """The paper's pipeline on CPU devices alone: sample each socket's FPM, FPM
    partition (bit-exact vs the oracle partitioner), arrangement (bit-exact vs
    the oracle), multiply (vs the oracle GEMM)."""
    if NCORES < 3:
        pytest.skip("needs 3 host cores")
    N, b = 512, 64
    n = N // b
    caps = [NCORES - NCORES // 3, NCORES // 3]
    sizes = [1, 4, 9, 16]
    with pkg.Context.local([CPU, CPU], sm_caps=caps) as ctx:
        models = [(sizes, ctx.sample(i, b, sizes, pkg.FPM_F32)[0]) for i in range(2)]
        d = pkg.fpm_partition(n * n, models)
        assert d == ofpm.partition(n * n, models)
        rects = pkg.colpart_arrange(n, d)
        assert rects == ofpm.arrange(n, d)
        A = synth.rect(3, N, 0, 0, N, N)
        B = synth.rect(4, N, 0, 0, N, N)
        C = np.empty((N, N), np.float32)
        ctx.run(A, B, C, N, b, rects, pkg.FPM_F32)
    assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


def test_cpu_device_options_and_errors():
    with pytest.raises(pkg.FpmError):
        pkg.Context.local([CPU], sm_caps=[NCORES + 1])          # more cores than the affinity mask
    with pkg.Context.local([CPU], sm_caps=[1]) as ctx:
        if NCORES > 1:
            ctx.set_device_option(0, "cpu_first_core", NCORES - 1)   # move the team to the last core
        with pytest.raises(pkg.FpmError):
            ctx.set_device_option(0, "cpu_first_core", NCORES)       # outside the mask: kept where it was
        with pytest.raises(pkg.FpmError):
            ctx.set_device_option(0, "c_cap_bytes", 1 << 20)         # GPU-only option
        N, b = 128, 32
        A = synth.rect(1, N, 0, 0, N, N)
        B = synth.rect(2, N, 0, 0, N, N)
        C = np.empty((N, N), np.float32)
        ctx.run(A, B, C, N, b, [(0, 0, 0, 4, 4)], pkg.FPM_F32)        # still works after the failed move
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


def test_sample_rects_and_operating_point_refinement():
    """fpm_sample_rects on a CPU device (any rectangle, speed attributed to
    x = h w) and the synchronised level correction (studies/refine.py, reading
    Q26) on two CPU devices: it terminates, every round's partition sums to T,
    and each refined model is its size-sweep model times one ratio (the shape
    is kept), the ratio = sampled / modelled speed at the operating point."""
    if NCORES < 2:
        pytest.skip("needs 2 host cores")
    from studies import refine as rf
    n, b = 12, 64
    with pkg.Context.local([CPU, CPU], sm_caps=[1, 1]) as ctx:
        sp, ci, reps = ctx.sample_rects(0, b, [(2, 3), (3, 2), (4, 4)], pkg.FPM_F32)
        assert len(sp) == 3 and all(s > 0 for s in sp) and all(r >= 5 for r in reps)
        sizes = [1, 4, 16]
        models = [(sizes, ctx.sample(i, b, sizes, pkg.FPM_F32)[0]) for i in range(2)]
        mods, hist, d, rects = rf.refine(ctx, n, b, models, rounds=3, concurrent=False)
        assert sum(d) == n * n and 1 <= len(hist) <= 3
        for h in hist:
            assert sum(h["d"]) == n * n
        # the returned partition is one that was timed: the converged one (last round) or
        # the candidate with the smallest measured makespan
        assert d in [h["d"] for h in hist]
        chosen = [h for h in hist if h["d"] == d][-1]
        assert chosen is hist[-1] or chosen["measured_makespan_rel"] == min(h["measured_makespan_rel"] for h in hist)
        for i in range(2):
            assert mods[i][0] == sizes   # the shape of the size sweep is kept: one ratio per device
            k = mods[i][1][0] / models[i][1][0]
            assert all(abs(a - k * s0) <= 1e-9 * a for a, s0 in zip(mods[i][1], models[i][1]))
        if chosen is hist[-1] and len(hist) < 3:   # converged: the models carry that round's levels
            for i in range(2):
                x = chosen["areas"][i]
                assert abs(pkg.fpm_model_speed(mods[i], x) - chosen["sampled_gflops"][i] * 1e9) <= \
                    1e-6 * pkg.fpm_model_speed(mods[i], x)


def test_cliff_areas_and_rescale():
    """Cliff bracketing: 1 GiB of FP32 C at b = 512 holds 1024 blocks (32 x 32);
    1025 = 25 x 41 is not nearly square, the smallest out-of-core area with a
    rectangle of aspect <= 2 is 1026 = 27 x 38.  rescale() keeps the other
    side of a cliff untouched."""
    from studies import refine as rf
    (x_in, r_in), (x_out, r_out) = rf.cliff_areas(1 << 30, 512)
    assert (x_in, r_in) == (1024, (32, 32))
    assert x_out > 1024 and r_out[0] * r_out[1] == x_out and r_out[1] / r_out[0] <= 2.0
    assert all(rf.near_square(x) is None for x in range(1025, x_out))
    m = ([1, 4, 1024, x_out, 2000], [1.0, 2.0, 3.0, 1.0, 1.0])
    xs, ss, k = rf.rescale(m, 2000, 0.5, split=1024)
    assert k == 0.5 and ss == [1.0, 2.0, 3.0, 0.5, 0.5]
    xs, ss, k = rf.rescale(m, 4, 4.0)
    assert k == 2.0 and ss == [2.0, 4.0, 6.0, 2.0, 2.0]


def test_refine_add_point():
    from studies import refine as rf
    assert rf.add_point(([1, 4, 9], [1.0, 2.0, 3.0]), 6, 2.5) == ([1, 4, 6, 9], [1.0, 2.0, 2.5, 3.0])
    assert rf.add_point(([1, 4], [1.0, 2.0]), 4, 5.0) == ([1, 4], [1.0, 5.0])
    assert rf.add_point(([4], [2.0]), 1, 1.0) == ([1, 4], [1.0, 2.0])
