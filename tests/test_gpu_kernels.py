"""Kernel-level parity on the GPU (through the C ABI): generator, operand split,
transpose, FP32 (F16X3 / TF32X3, 1- and 2-CTA) and FP64 rank-b updates vs the oracle."""
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
    torch.cuda.set_device(0)
    yield
    torch.cuda.synchronize()


def T(x):
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


@pytest.mark.parametrize("dt", [pkg.FPM_F32, pkg.FPM_F64])
@pytest.mark.parametrize("dist", [pkg.FPM_DIST_PM1, pkg.FPM_DIST_INT])
def test_fill_synthetic_bit_exact(dt, dist):
    npdt = np.float32 if dt == pkg.FPM_F32 else np.float64
    out = torch.zeros((40, 56), dtype=torch.float32 if dt == pkg.FPM_F32 else torch.float64, device="cuda")
    pkg.k_fill_synthetic(out, dt, 56, 7, 300, 17, 33, 40, 50, dist)
    torch.cuda.synchronize()
    ref = synth.rect(7, 300, 17, 33, 40, 50, dist, npdt)
    got = out.cpu().numpy()
    assert np.array_equal(got[:, :50], ref)
    assert np.all(got[:, 50:] == 0)


def _scaled_rows(rows, K, seed):
    x = synth.rect(seed, 4096, 0, 0, rows, K).astype(np.float64)
    rng = np.random.default_rng(seed)
    x *= 10.0 ** rng.uniform(-6, 6, size=(rows, 1))
    x[rows // 3] = 0.0
    return x.astype(np.float32)


def test_split_f16x3_reconstructs():
    rows, K = 301, 192
    x = _scaled_rows(rows, K, 3)
    src = T(x)
    hi = torch.empty((rows, K), dtype=torch.float16, device="cuda")
    lo = torch.empty_like(hi)
    inv = torch.empty(rows, dtype=torch.float32, device="cuda")
    pkg.k_split_f32(src, K, rows, K, pkg.SCHEME_F16X3, hi, lo, inv)
    torch.cuda.synchronize()
    h = hi.double().cpu().numpy()
    l = lo.double().cpu().numpy()
    s = inv.double().cpu().numpy()
    m, e = np.frexp(s)
    assert np.all(m == 0.5)                       # inverse scales are powers of two
    rec = (h + l) * s[:, None]
    rowmax = np.abs(x).max(axis=1, keepdims=True).astype(np.float64)
    err = np.abs(rec - x.astype(np.float64))
    assert np.all(err <= 2.0 ** -21 * rowmax + 1e-300)
    nz = rowmax[:, 0] > 0
    hm = np.abs(h).max(axis=1)
    assert np.all(hm[nz] >= 2.0 ** 14) and np.all(hm[nz] <= 2.0 ** 15)


def _np_split_f16(x):
    """Reading Q15 written out in numpy: per row, 2^s puts the row max in
    [2^14, 2^15); h0 = fp16_rn(x 2^s), h1 = fp16_rn(x 2^s - h0) in fp32."""
    m = np.abs(x).max(axis=1)
    _, e = np.frexp(m)
    s = np.where(m > 0, np.clip(15 - e, -126, 127), 0).astype(np.int32)
    xs = (x * np.ldexp(np.float32(1), s)[:, None]).astype(np.float32)
    h0 = xs.astype(np.float16)
    h1 = (xs - h0.astype(np.float32)).astype(np.float16)
    return h0, h1, np.ldexp(np.float32(1), -s).astype(np.float32)


def test_split_rows_f16x3_bit_exact_vs_numpy():
    rows, K = 130, 256
    x = _scaled_rows(rows, K, 5)
    hi = torch.empty((rows, K), dtype=torch.float16, device="cuda")
    lo = torch.empty_like(hi)
    inv = torch.empty(rows, dtype=torch.float32, device="cuda")
    pkg.k_split_f32(T(x), K, rows, K, pkg.SCHEME_F16X3, hi, lo, inv)
    torch.cuda.synchronize()
    h0, h1, s = _np_split_f16(x)
    assert np.array_equal(hi.cpu().numpy().view(np.uint16), h0.view(np.uint16))
    assert np.array_equal(lo.cpu().numpy().view(np.uint16), h1.view(np.uint16))
    assert np.array_equal(inv.cpu().numpy(), s)


@pytest.mark.parametrize("K,W,ld", [(64, 256, 256), (512, 1000, 1004), (32, 4, 8), (520, 388, 392)])
def test_split_cols_bit_exact_vs_numpy(K, W, ld):
    """B pivot row K x W -> split halves of its transpose (W x K)."""
    src = _scaled_rows(W, K, 6).T.copy()           # K x W with per-column scales
    src = np.pad(src, ((0, 0), (0, ld - W)), constant_values=7.0)
    for scheme in (pkg.SCHEME_F16X3, pkg.SCHEME_TF32X3):
        odt = torch.float16 if scheme == pkg.SCHEME_F16X3 else torch.float32
        hi = torch.empty((W, K), dtype=odt, device="cuda")
        lo = torch.empty_like(hi)
        inv = torch.empty(W, dtype=torch.float32, device="cuda")
        pkg.k_split_cols_f32(T(src), ld, K, W, scheme, hi, lo, inv)
        torch.cuda.synchronize()
        xt = np.ascontiguousarray(src[:, :W].T)
        if scheme == pkg.SCHEME_F16X3:
            h0, h1, s = _np_split_f16(xt)
            assert np.array_equal(hi.cpu().numpy().view(np.uint16), h0.view(np.uint16))
            assert np.array_equal(lo.cpu().numpy().view(np.uint16), h1.view(np.uint16))
            assert np.array_equal(inv.cpu().numpy(), s)
        else:
            hb = hi.cpu().numpy()
            assert np.all(hb.view(np.uint32) & 0x1FFF == 0)
            rec = hb.astype(np.float64) + lo.cpu().numpy().astype(np.float64)
            assert np.all(np.abs(rec - xt) <= 2.0 ** -21 * np.abs(xt.astype(np.float64)) + 1e-300)


def test_split_tf32x3_reconstructs():
    rows, K = 257, 96
    x = _scaled_rows(rows, K, 4)
    src = T(x)
    hi = torch.empty((rows, K), dtype=torch.float32, device="cuda")
    lo = torch.empty_like(hi)
    pkg.k_split_f32(src, K, rows, K, pkg.SCHEME_TF32X3, hi, lo, None)
    torch.cuda.synchronize()
    hb = hi.cpu().numpy().view(np.uint32)
    lb = lo.cpu().numpy().view(np.uint32)
    assert np.all(hb & 0x1FFF == 0) and np.all(lb & 0x1FFF == 0)
    rec = hi.double().cpu().numpy() + lo.double().cpu().numpy()
    assert np.all(np.abs(rec - x) <= 2.0 ** -21 * np.abs(x.astype(np.float64)) + 1e-300)


@pytest.mark.parametrize("dt", [pkg.FPM_F32, pkg.FPM_F64])
@pytest.mark.parametrize("rows,cols", [(64, 96), (1, 33), (130, 1000), (512, 64)])
def test_transpose_bit_exact(dt, rows, cols):
    npdt = np.float32 if dt == pkg.FPM_F32 else np.float64
    ld = cols + 5
    x = synth.rect(9, 2048, 0, 0, rows, ld, dtype=npdt)
    out = torch.empty((cols, rows), dtype=torch.float32 if dt == pkg.FPM_F32 else torch.float64, device="cuda")
    pkg.k_transpose(T(x), dt, ld, rows, cols, out)
    torch.cuda.synchronize()
    assert np.array_equal(out.cpu().numpy(), x[:, :cols].T)


KCFG = ["1", "2v0", "2v1", "2v2", "2v3", "2v4", "2v5"]   # cta_group 1; cta_group 2 with smem variants 0..5 (5: reduce-add C)


def _update_f32(A, B, C0, scheme, cg, num_sms=0, accumulate=True):
    cg = str(cg)
    variant = int(cg[2]) if "v" in cg else 1
    cg = int(cg[0])
    M, K = A.shape
    Nc = B.shape[1]
    half = scheme == pkg.SCHEME_F16X3
    odt = torch.float16 if half else torch.float32
    Bt = np.ascontiguousarray(B.T)
    a_hi = torch.empty((M, K), dtype=odt, device="cuda"); a_lo = torch.empty_like(a_hi)
    b_hi = torch.empty((Nc, K), dtype=odt, device="cuda"); b_lo = torch.empty_like(b_hi)
    sa = torch.empty(M, dtype=torch.float32, device="cuda")
    sb = torch.empty(Nc, dtype=torch.float32, device="cuda")
    pkg.k_split_f32(T(A), K, M, K, scheme, a_hi, a_lo, sa)
    if Nc % 4 == 0:   # the product path: split of the transposed B pivot row in one pass
        pkg.k_split_cols_f32(T(B), Nc, K, Nc, scheme, b_hi, b_lo, sb)
    else:
        pkg.k_split_f32(T(Bt), K, Nc, K, scheme, b_hi, b_lo, sb)
    C = T(C0)
    pkg.k_update_f32(a_hi, a_lo, b_hi, b_lo, sa if half else None, sb if half else None, C, M, Nc, K,
                     C0.shape[1], scheme, cg, num_sms, accumulate, variant)
    torch.cuda.synchronize()
    return C.cpu().numpy()


SHAPES = [(128, 256, 64), (300, 520, 96), (1000, 1000, 512), (64, 40, 32), (1, 8, 32), (2048, 2304, 1024),
          (777, 264, 160)]


@pytest.mark.parametrize("scheme", [pkg.SCHEME_F16X3, pkg.SCHEME_TF32X3])
@pytest.mark.parametrize("cg", KCFG)
@pytest.mark.parametrize("M,Nc,K", SHAPES)
def test_update_f32_random(scheme, cg, M, Nc, K):
    A = synth.rect(1, 4096, 0, 0, M, K)
    B = synth.rect(2, 4096, 0, 0, K, Nc)
    C0 = synth.rect(3, 4096, 0, 0, M, Nc)
    C = _update_f32(A, B, C0, scheme, cg)
    ref = C0.astype(np.float64) + og.gemm(A, B)
    err = og.rel_fro(C, ref)
    assert err <= 1e-5, err


@pytest.mark.parametrize("scheme", [pkg.SCHEME_F16X3, pkg.SCHEME_TF32X3])
@pytest.mark.parametrize("cg", KCFG)
def test_update_f32_integer_exact(scheme, cg):
    M, Nc, K = 520, 776, 512
    A = synth.rect(4, 4096, 0, 0, M, K, synth.DIST_INT)
    B = synth.rect(5, 4096, 0, 0, K, Nc, synth.DIST_INT)
    C0 = synth.rect(6, 4096, 0, 0, M, Nc, synth.DIST_INT)
    C = _update_f32(A, B, C0, scheme, cg)
    assert np.array_equal(C.astype(np.float64), C0.astype(np.float64) + og.gemm(A, B))


@pytest.mark.parametrize("scheme", [pkg.SCHEME_F16X3, pkg.SCHEME_TF32X3])
@pytest.mark.parametrize("cg", KCFG)
def test_update_f32_overwrite_ignores_c(scheme, cg):
    """accumulate = 0 (iteration 0): C = A B, the old C (NaN here) is never read."""
    M, Nc, K = 700, 520, 128
    A = synth.rect(1, 4096, 0, 0, M, K)
    B = synth.rect(2, 4096, 0, 0, K, Nc)
    C = _update_f32(A, B, np.full((M, Nc), np.nan, np.float32), scheme, cg, accumulate=False)
    assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5
    Ai = synth.rect(4, 4096, 0, 0, M, K, synth.DIST_INT)
    Bi = synth.rect(5, 4096, 0, 0, K, Nc, synth.DIST_INT)
    Ci = _update_f32(Ai, Bi, np.full((M, Nc), np.nan, np.float32), scheme, cg, accumulate=False)
    assert np.array_equal(Ci.astype(np.float64), og.gemm(Ai, Bi))


def test_update_f32_identity_and_sm_cap():
    K = 256
    A = synth.rect(7, 4096, 0, 0, 384, K, synth.DIST_INT)
    I = np.eye(K, dtype=np.float32)
    C = _update_f32(A, I, np.zeros((384, K), np.float32), pkg.SCHEME_F16X3, 2, num_sms=16)
    assert np.array_equal(C, A)


def test_update_f32_wide_dynamic_range():
    """Per-row power-of-two scaling keeps FP32-class accuracy for rows of very
    different magnitude (reading Q15)."""
    M, Nc, K = 256, 256, 256
    A = _scaled_rows(M, K, 8)
    B = _scaled_rows(Nc, K, 9).T.copy()
    C = _update_f32(A, B, np.zeros((M, Nc), np.float32), pkg.SCHEME_F16X3, 2)
    ref = og.gemm(A, B)
    # row- and column-wise relative error (each row/col has its own scale)
    den = np.abs(A).astype(np.float64).max(1, keepdims=True) * np.abs(B).astype(np.float64).max(0, keepdims=True)
    den[den == 0] = 1.0
    assert np.max(np.abs(C - ref) / den) <= K * 2.0 ** -20


@pytest.mark.parametrize("M,Nc,K", [(64, 64, 64), (300, 520, 96), (513, 130, 8), (1, 1, 16)])
def test_update_f64(M, Nc, K):
    A = synth.rect(1, 4096, 0, 0, M, K, dtype=np.float64)
    B = synth.rect(2, 4096, 0, 0, K, Nc, dtype=np.float64)
    C0 = synth.rect(3, 4096, 0, 0, M, Nc, dtype=np.float64)
    C = T(C0)
    pkg.k_update_f64(T(A), K, T(np.ascontiguousarray(B.T)), C, M, Nc, K, Nc)
    torch.cuda.synchronize()
    ref = C0 + og.gemm(A, B)
    assert og.rel_fro(C.cpu().numpy(), ref) <= 1e-12
    Ai = synth.rect(4, 4096, 0, 0, M, K, synth.DIST_INT, np.float64)
    Bi = synth.rect(5, 4096, 0, 0, K, Nc, synth.DIST_INT, np.float64)
    Ci = torch.full((M, Nc), float("nan"), dtype=torch.float64, device="cuda")
    pkg.k_update_f64(T(Ai), K, T(np.ascontiguousarray(Bi.T)), Ci, M, Nc, K, Nc, accumulate=False)
    torch.cuda.synchronize()
    assert np.array_equal(Ci.cpu().numpy(), og.gemm(Ai, Bi))
