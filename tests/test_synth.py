"""The shared input generator: distribution, exactness and rect consistency."""
import numpy as np

import synth


def test_pm1_range_and_exactness():
    x = synth.matrix_pm1(1, 256)
    assert x.dtype == np.float32
    assert x.min() >= -1.0 and x.max() < 1.0
    # values are k * 2^-23 - 1: exact multiples of 2^-23
    k = (x.astype(np.float64) + 1.0) * 2.0 ** 23
    assert np.array_equal(k, np.round(k))
    assert abs(float(x.mean())) < 0.01
    assert abs(float(x.var()) - 1.0 / 3.0) < 0.01


def test_int_range():
    x = synth.matrix_int(3, 200)
    assert x.min() == -8 and x.max() == 8
    assert np.array_equal(x, np.round(x))


def test_rect_is_window_of_global():
    N = 96
    full = synth.matrix_pm1(7, N)
    r = synth.rect(7, N, 17, 33, 40, 21)
    assert np.array_equal(r, full[17:57, 33:54])


def test_known_hash_values():
    # splitmix64 finaliser of key + (idx+1)*golden, hand-computed with Python ints
    def ref(seed, idx):
        M = (1 << 64) - 1
        z = (seed * 0xD1B54A32D192ED03 + (idx + 1) * 0x9E3779B97F4A7C15) & M
        z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
        z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
        return z ^ (z >> 31)
    idx = np.array([0, 1, 2, 12345678901], dtype=np.uint64)
    got = synth.hash64(42, idx)
    assert [int(v) for v in got] == [ref(42, int(i)) for i in idx]


def test_seeds_differ():
    assert not np.array_equal(synth.matrix_pm1(1, 32), synth.matrix_pm1(2, 32))


def test_stress_distributions_moments_and_windows():
    """Gaussian / signed-lognormal stress inputs: right moments, and a window of
    the global matrix equals the same entries of the whole matrix (counter-based)."""
    N = 600
    g = synth.gaussian(7, N, 0, 0, N, N, np.float64)
    assert abs(g.mean()) < 0.01 and abs(g.std() - 1.0) < 0.01
    assert abs(np.mean(g ** 4) - 3.0) < 0.1            # Gaussian kurtosis
    np.testing.assert_array_equal(synth.gaussian(7, N, 100, 50, 30, 40, np.float64), g[100:130, 50:90])
    lg = synth.lognormal_signed(7, N, 0, 0, N, N, 1.0, np.float64)
    mag = np.log(np.abs(lg))
    assert abs(mag.mean()) < 0.01 and abs(mag.std() - 1.0) < 0.01
    assert abs((lg > 0).mean() - 0.5) < 0.01
    np.testing.assert_array_equal(synth.lognormal_signed(7, N, 5, 9, 3, 4, 1.0, np.float64), lg[5:8, 9:13])
