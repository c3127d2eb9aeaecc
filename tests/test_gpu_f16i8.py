"""F16I8, the opt-in (not FP32-class) FP32 scheme of the rank-b update (reading Q15b):
x 2^e = h0 + h1 (h0 fp16), int8 codes q = clamp(rint(x 2^e / 256), +-127) and
l = rint(8 h1); C += 2^-(ea+eb) (h0a h0b' + 32 (qa lb' + la qb')) with the fp16
product on kind::f16 and the two cross terms as ONE kind::i8 product.

Split kernels bit-exact against the scheme written out in numpy; the update
against the oracle (FP64 triple loop) within the FP32 tolerance 1e-5,
bit-exact on integer inputs (where h1 = 0), through the C ABI."""
import numpy as np
import pytest

import synth
from oracle import gemm as og

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
import paper_conf_cluster_zhongrl12_b200 as pkg  # noqa: E402

S = pkg.SCHEME_F16I8


@pytest.fixture(autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    torch.cuda.set_device(0)
    yield
    torch.cuda.synchronize()


def T(x):
    return torch.from_numpy(np.ascontiguousarray(x)).cuda()


def _scaled_rows(rows, K, seed):
    x = synth.rect(seed, 4096, 0, 0, rows, K).astype(np.float64)
    rng = np.random.default_rng(seed)
    x *= 10.0 ** rng.uniform(-6, 6, size=(rows, 1))
    x[rows // 3] = 0.0
    return x.astype(np.float32)


def _np_f16i8(x, b_side):
    """The scheme written out: per row the F16X3 scale 2^s (row max in
    [2^14, 2^15)), h0 = fp16_rn(x 2^s), q = clamp(rint(x 2^s / 256), +-127),
    l = rint(8 (x 2^s - h0)); int8 rows of 128 bytes per 64-wide k-block,
    [q | l] for A, [l | q] for B^T."""
    rows, K = x.shape
    m = np.abs(x).max(axis=1)
    _, e = np.frexp(m)
    s = np.where(m > 0, np.clip(15 - e, -126, 127), 0).astype(np.int32)
    xs = (x * np.ldexp(np.float32(1), s)[:, None]).astype(np.float32)
    h0 = xs.astype(np.float16)
    q = np.clip(np.rint(xs / np.float32(256)), -127, 127).astype(np.int8)
    l = np.rint((xs - h0.astype(np.float32)) * np.float32(8)).astype(np.int8)
    assert np.abs(l.astype(np.int32)).max(initial=0) <= 64
    first, second = (l, q) if b_side else (q, l)
    codes = np.empty((rows, K // 64, 128), np.int8)
    codes[:, :, :64] = first.reshape(rows, K // 64, 64)
    codes[:, :, 64:] = second.reshape(rows, K // 64, 64)
    return h0, codes.reshape(rows, 2 * K), np.ldexp(np.float32(1), -s).astype(np.float32)


@pytest.mark.parametrize("rows,K", [(130, 256), (301, 64), (8, 1024)])
def test_split_rows_f16i8_bit_exact_vs_numpy(rows, K):
    x = _scaled_rows(rows, K, 5)
    hi = torch.empty((rows, K), dtype=torch.float16, device="cuda")
    lo = torch.empty((rows, 2 * K), dtype=torch.int8, device="cuda")
    inv = torch.empty(rows, dtype=torch.float32, device="cuda")
    pkg.k_split_f32(T(x), K, rows, K, S, hi, lo, inv)
    torch.cuda.synchronize()
    h0, codes, s = _np_f16i8(x, b_side=False)
    assert np.array_equal(hi.cpu().numpy().view(np.uint16), h0.view(np.uint16))
    assert np.array_equal(lo.cpu().numpy(), codes)
    assert np.array_equal(inv.cpu().numpy(), s)


@pytest.mark.parametrize("K,W,ld", [(64, 256, 256), (512, 1000, 1004), (128, 4, 8)])
def test_split_cols_f16i8_bit_exact_vs_numpy(K, W, ld):
    """B pivot row K x W -> fp16 h0 and int8 codes of its transpose (W x K)."""
    src = _scaled_rows(W, K, 6).T.copy()
    src = np.pad(src, ((0, 0), (0, ld - W)), constant_values=7.0)
    hi = torch.empty((W, K), dtype=torch.float16, device="cuda")
    lo = torch.empty((W, 2 * K), dtype=torch.int8, device="cuda")
    inv = torch.empty(W, dtype=torch.float32, device="cuda")
    pkg.k_split_cols_f32(T(src), ld, K, W, S, hi, lo, inv)
    torch.cuda.synchronize()
    h0, codes, s = _np_f16i8(np.ascontiguousarray(src[:, :W].T), b_side=True)
    assert np.array_equal(hi.cpu().numpy().view(np.uint16), h0.view(np.uint16))
    assert np.array_equal(lo.cpu().numpy(), codes)
    assert np.array_equal(inv.cpu().numpy(), s)


def _update(A, B, C0, variant=-1, num_sms=0, accumulate=True):
    M, K = A.shape
    Nc = B.shape[1]
    a_hi = torch.empty((M, K), dtype=torch.float16, device="cuda")
    a_8 = torch.empty((M, 2 * K), dtype=torch.int8, device="cuda")
    b_hi = torch.empty((Nc, K), dtype=torch.float16, device="cuda")
    b_8 = torch.empty((Nc, 2 * K), dtype=torch.int8, device="cuda")
    sa = torch.empty(M, dtype=torch.float32, device="cuda")
    sb = torch.empty(Nc, dtype=torch.float32, device="cuda")
    pkg.k_split_f32(T(A), K, M, K, S, a_hi, a_8, sa)
    pkg.k_split_cols_f32(T(B), Nc, K, Nc, S, b_hi, b_8, sb)
    C = T(C0)
    pkg.k_update_f32(a_hi, a_8, b_hi, b_8, sa, sb, C, M, Nc, K, C0.shape[1], S, 2, num_sms, accumulate, variant)
    torch.cuda.synchronize()
    return C.cpu().numpy()


SHAPES = [(128, 256, 64), (300, 520, 128), (1000, 1000, 512), (64, 40, 64), (1, 8, 64), (2048, 2304, 1024),
          (777, 264, 192), (520, 1032, 2048)]


@pytest.mark.parametrize("variant", [-1, 0, 1, 2, 4, 5, 6])
@pytest.mark.parametrize("M,Nc,K", SHAPES)
def test_update_f16i8_random(variant, M, Nc, K):
    A = synth.rect(1, 4096, 0, 0, M, K)
    B = synth.rect(2, 4096, 0, 0, K, Nc)
    C0 = synth.rect(3, 4096, 0, 0, M, Nc)
    C = _update(A, B, C0, variant)
    ref = C0.astype(np.float64) + og.gemm(A, B)
    assert og.rel_fro(C, ref) <= 1e-5


@pytest.mark.parametrize("variant", [-1, 0, 1, 2, 4, 5, 6])
def test_update_f16i8_integer_exact(variant):
    M, Nc, K = 520, 776, 512
    A = synth.rect(4, 4096, 0, 0, M, K, synth.DIST_INT)
    B = synth.rect(5, 4096, 0, 0, K, Nc, synth.DIST_INT)
    C0 = synth.rect(6, 4096, 0, 0, M, Nc, synth.DIST_INT)
    C = _update(A, B, C0, variant)
    assert np.array_equal(C.astype(np.float64), C0.astype(np.float64) + og.gemm(A, B))


def test_update_f16i8_overwrite_ignores_c():
    M, Nc, K = 700, 520, 128
    A = synth.rect(1, 4096, 0, 0, M, K)
    B = synth.rect(2, 4096, 0, 0, K, Nc)
    C = _update(A, B, np.full((M, Nc), np.nan, np.float32), accumulate=False)
    assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5
    Ai = synth.rect(4, 4096, 0, 0, M, K, synth.DIST_INT)
    Bi = synth.rect(5, 4096, 0, 0, K, Nc, synth.DIST_INT)
    Ci = _update(Ai, Bi, np.full((M, Nc), np.nan, np.float32), accumulate=False)
    assert np.array_equal(Ci.astype(np.float64), og.gemm(Ai, Bi))


def test_update_f16i8_identity_and_sm_cap():
    K = 256
    A = synth.rect(7, 4096, 0, 0, 384, K, synth.DIST_INT)
    C = _update(A, np.eye(K, dtype=np.float32), np.zeros((384, K), np.float32), num_sms=16)
    assert np.array_equal(C, A)


def test_update_f16i8_wide_dynamic_range():
    """Rows / columns spanning 12 decades: the per-row scales keep the error
    relative to each row's and column's own magnitude."""
    M, Nc, K = 256, 256, 256
    A = _scaled_rows(M, K, 8)
    B = _scaled_rows(Nc, K, 9).T.copy()
    C = _update(A, B, np.zeros((M, Nc), np.float32))
    ref = og.gemm(A, B)
    den = np.abs(A).astype(np.float64).max(1, keepdims=True) * np.abs(B).astype(np.float64).max(0, keepdims=True)
    den[den == 0] = 1.0
    # per product: |h0 - 256 q| <= 128 times |h1| <= 8, twice, plus fp32 accumulation
    assert np.max(np.abs(C - ref) / den) <= K * 2.0 ** -16


def test_update_f16i8_rejects_ragged_k():
    M, Nc, K = 64, 64, 96
    z = torch.zeros((M, 2 * K), dtype=torch.int8, device="cuda")
    h = torch.zeros((M, K), dtype=torch.float16, device="cuda")
    s = torch.ones(M, device="cuda")
    C = torch.zeros((M, Nc), device="cuda")
    with pytest.raises(pkg.FpmError):
        pkg.k_update_f32(h, z, h, z, s, s, C, M, Nc, K, Nc, S, 2)


def test_update_f16i8_intra_row_dynamic_range_is_normwise():
    """Entries spanning 2^0 .. 2^-20 inside each row / column: F16I8's error is
    bounded relative to the row and column maxima (reading Q15b), F16X3's
    relative to the elements -- the documented difference between the two."""
    M, Nc, K = 256, 320, 512
    rng = np.random.default_rng(11)
    A = (synth.rect(1, 4096, 0, 0, M, K).astype(np.float64) * 2.0 ** -rng.integers(0, 21, (M, K))).astype(np.float32)
    B = (synth.rect(2, 4096, 0, 0, K, Nc).astype(np.float64) * 2.0 ** -rng.integers(0, 21, (K, Nc))).astype(np.float32)
    C = _update(A, B, np.zeros((M, Nc), np.float32))
    ref = og.gemm(A, B)
    den = np.abs(A).astype(np.float64).max(1, keepdims=True) * np.abs(B).astype(np.float64).max(0, keepdims=True)
    assert np.max(np.abs(C - ref) / den) <= K * 2.0 ** -16


def test_prof_counters_count_tiles_and_reset():
    """fpm_k_prof: the MMA issuer's counters see every tile of a profiled launch,
    stay at zero while disabled, and reset on enable."""
    M, Nc, K = 512, 768, 128
    A = synth.rect(1, 4096, 0, 0, M, K)
    B = synth.rect(2, 4096, 0, 0, K, Nc)
    pkg.k_prof(1)
    _update(A, B, np.zeros((M, Nc), np.float32))
    pr = pkg.k_prof(2)
    pkg.k_prof(0)
    assert pr["tiles"] == (M // 256) * (Nc // 256)          # 256 x 256 tiles, one count per CTA pair
    assert 0 < pr["tmem_wait"] + pr["operand_wait"] <= pr["issuer"]
    pkg.k_prof(1)
    pkg.k_prof(0)
    _update(A, B, np.zeros((M, Nc), np.float32))             # disabled: not counted
    assert pkg.k_prof(2)["tiles"] == 0
