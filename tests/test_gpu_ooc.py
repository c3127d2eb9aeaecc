"""Out-of-core C_i (PAPER.md P:34-40 GPU kernel versions
2-3): a device whose C_i exceeds its memory cap keeps C_i in pinned host
memory and streams it through two band buffers every update.  Parity with the
oracle, exact byte accounting, and the speed-function cliff (Table III)."""
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


def _inputs(N, dt, dist=synth.DIST_PM1, seeds=(1, 2)):
    npdt = np.float32 if dt == pkg.FPM_F32 else np.float64
    A = synth.rect(seeds[0], N, 0, 0, N, N, dist, npdt)
    B = synth.rect(seeds[1], N, 0, 0, N, N, dist, npdt)
    return A, B, np.full((N, N), np.nan, dtype=npdt)


def _cap_for_band_rows(rows, W, es, R=2):
    """c_cap_bytes that gives bands of `rows` rows (R buffers of rows x W)."""
    return R * rows * W * es


def _expected_ooc_bytes(H, W, es, band_rows, updates, keep, R=2):
    """Host <-> device C bytes of one k-loop, written from P:34 directly: every
    update moves each band in (not the first update: it overwrites) and out;
    with `keep` the order reverses every other update and the last R bands of
    an update (the paper: two) stay on the device for the next one (not after
    the last)."""
    rows = [min(band_rows, H - r0) for r0 in range(0, H, band_rows)]
    nb, nkeep = len(rows), min(R, len(rows))
    total = 0
    for g in range(updates):
        order = list(range(nb))[::-1] if keep and g % 2 else list(range(nb))
        head = set(order[:nkeep]) if keep and g > 0 else set()
        tail = set(order[-nkeep:]) if keep and g + 1 < updates else set()
        total += sum(rows[j] for j in order if g > 0 and j not in head)
        total += sum(rows[j] for j in order if j not in tail)
    return total * W * es


@pytest.mark.parametrize("dt,tol", [(pkg.FPM_F32, 1e-5), (pkg.FPM_F64, 1e-12)])
@pytest.mark.parametrize("band_rows", [256, 512, 0])
@pytest.mark.parametrize("keep,R", [(1, 2), (0, 2), (1, 3), (1, 8)])
def test_ooc_device_parity(dt, tol, band_rows, keep, R):
    """Device 0 out of core with 1, 3 or 5 bands (ragged), device 1 resident;
    R band buffers (the paper's two, and rings of 3 and 8)."""
    N, b = 1440, 96          # rect 0 is 1056 x 1440: bands 4 x 256 + 32, 2 x 512 + 32
    n = N // b
    rects = pkg.colpart_arrange(n, [n * n - 60, 60])
    if band_rows == 0:       # 192-row rect 0 below the 256-row band minimum: one band
        rects = [(0, 0, 0, 2, n), (0, 2, 0, n - 2, n)]
    es = 4 if dt == pkg.FPM_F32 else 8
    r0 = rects[0]
    H0, W0 = r0[3] * b, r0[4] * b
    A, B, C = _inputs(N, dt)
    cap = _cap_for_band_rows(band_rows, W0, es, R) if band_rows else 1
    with pkg.Context.local([0, 0]) as ctx:
        ctx.set_option("ooc_keep", keep)
        ctx.set_option("ooc_buffers", R)
        ctx.set_device_option(0, "c_cap_bytes", cap)
        st = ctx.run(A, B, C, N, b, rects, dt)
    assert og.rel_fro(C, og.gemm(A, B)) <= tol
    if cap >= H0 * W0 * es:           # C_0 fits the cap: stays resident
        assert st.ooc_devices == 0 and st.ooc_bytes == 0
        return
    assert st.ooc_devices == 1
    br = max(band_rows, 256)
    assert st.ooc_bytes == _expected_ooc_bytes(H0, W0, es, br, st.updates, keep, R)
    if not keep:
        assert st.ooc_bytes == H0 * W0 * es * (2 * st.updates - 1)
    nb = -(-H0 // br)
    assert st.kernel_launches >= st.updates * (nb + 1)


@pytest.mark.parametrize("fuse", [1, 2, 3])
def test_ooc_all_devices_integer_exact(fuse):
    """Integer inputs: bit-exact products with every device out of core and
    fused pivot groups (the band split must not change a single sum)."""
    N, b = 1024, 64
    n = N // b
    rects = pkg.colpart_arrange(n, [100, 80, 76])
    for dt, keep, R in ((pkg.FPM_F32, 1, 2), (pkg.FPM_F64, 1, 2), (pkg.FPM_F32, 0, 2), (pkg.FPM_F32, 1, 3)):
        A, B, C = _inputs(N, dt, dist=synth.DIST_INT, seeds=(11, 12))
        with pkg.Context.local([0, 0, 0]) as ctx:
            ctx.set_option("fuse", fuse)
            ctx.set_option("ooc_keep", keep)
            ctx.set_option("ooc_buffers", R)
            for i in range(3):
                ctx.set_device_option(i, "c_cap_bytes", 1)  # minimum bands: 256 rows
            st = ctx.run(A, B, C, N, b, rects, dt)
        assert np.array_equal(C.astype(np.float64), og.gemm(A, B))
        live = sum(1 << i for i, r in enumerate(rects) if r[3] * r[4] > 0)
        assert st.ooc_devices == live


def test_ooc_compute_download_block_and_reuse():
    """fill_synthetic + compute + download / download_block with an out-of-core
    device, then the cap lifted on the same context (C_i back in core)."""
    N, b = 1024, 128
    n = N // b
    rects = pkg.colpart_arrange(n, [40, 24])
    A = synth.rect(5, N, 0, 0, N, N)
    B = synth.rect(6, N, 0, 0, N, N)
    ref = og.gemm(A, B)
    with pkg.Context.local([0, 0]) as ctx:
        ctx.set_device_option(1, "c_cap_bytes", 1 << 20)
        ctx.setup(N, b, rects)
        ctx.fill_synthetic(5, 6)
        st = ctx.compute()
        assert st.ooc_devices == 2
        C = np.full((N, N), np.nan, np.float32)
        ctx.download(C, N)
        assert og.rel_fro(C, ref) <= 1e-5
        r1 = rects[1]
        R0, C0 = r1[1] * b, r1[2] * b
        blk = ctx.download_block(R0 + 3, C0 + 5, 17, 33)
        assert og.rel_fro(blk, ref[R0 + 3:R0 + 20, C0 + 5:C0 + 38]) <= 1e-5
        ctx.compute()                                   # second run on the same host C_i
        C2 = np.full((N, N), np.nan, np.float32)
        ctx.download(C2, N)
        assert np.array_equal(C, C2)
        ctx.set_device_option(1, "c_cap_bytes", 0)      # lift the cap: resident again
        ctx.setup(N, b, rects)
        ctx.fill_synthetic(5, 6)
        assert ctx.compute().ooc_devices == 0


def test_ooc_cap_not_exceeded_stays_resident():
    N, b = 512, 64
    with pkg.Context.local([0]) as ctx:
        ctx.set_device_option(0, "c_cap_bytes", N * N * 4)   # exactly fits
        A, B, C = _inputs(N, pkg.FPM_F32)
        st = ctx.run(A, B, C, N, b, [(0, 0, 0, N // b, N // b)], pkg.FPM_F32)
        assert st.ooc_devices == 0 and st.ooc_bytes == 0
        assert og.rel_fro(C, og.gemm(A, B)) <= 1e-5


def test_device_option_errors():
    with pkg.Context.local([0]) as ctx:
        with pytest.raises(pkg.FpmError):
            ctx.set_device_option(1, "c_cap_bytes", 1)      # no such device
        with pytest.raises(pkg.FpmError):
            ctx.set_device_option(0, "c_cap", 1)            # unknown key
        with pytest.raises(pkg.FpmError):
            ctx.set_device_option(0, "c_cap_bytes", -1)
        for bad in (1, 17):
            with pytest.raises(pkg.FpmError):
                ctx.set_option("ooc_buffers", bad)


def test_fpm_sample_shows_memory_cliff():
    """The speed function of a memory-capped device drops once C no longer fits
    ("the speed ... drops dramatically"; reading in DESIGN.md)."""
    b = 512
    with pkg.Context.local([0]) as ctx:
        L_fit = 8 * b
        ctx.set_device_option(0, "c_cap_bytes", L_fit * L_fit * 4)
        sizes = [36, 64, 100, 144]                          # L = 6b, 8b (fits), 10b, 12b (out of core)
        sp, _, reps = ctx.sample(0, b, sizes, pkg.FPM_F32)
        assert all(s > 0 for s in sp)
        assert sp[2] < 0.5 * sp[1] and sp[3] < 0.5 * sp[1]
        sp64, _, _ = ctx.sample(0, 64, [4, 1024], pkg.FPM_F64)  # 128 x 128 fits, 2048 x 2048 does not
        assert all(s > 0 for s in sp64)
