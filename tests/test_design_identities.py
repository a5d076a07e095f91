"""Host checks of the arithmetic identities the CUDA path relies on to
restructure work without changing a single bit.

These run numpy fp64 (IEEE, round-to-nearest-even) on CPU; the GPU parity
tests then confirm the kernels end to end (dt history bitwise).
"""
import numpy as np


def _logu(rng, lo, hi, n):
    return np.exp(rng.uniform(np.log(lo), np.log(hi), n))


def test_min_of_rounded_quotients_is_quotient_of_extreme():
    # DtAcc (clover_kernels.cuh): min_i RN(A / d_i) == RN(A / max_i d_i)
    rng = np.random.default_rng(11)
    for trial in range(200):
        A = float(_logu(rng, 1e-6, 1e3, 1)[0])
        n = int(rng.integers(1, 64))
        if trial % 3 == 0:  # near-ties: d differing in the last few ulps
            d = np.nextafter(np.full(n, _logu(rng, 1e-3, 1e3, 1)[0]), np.inf)
            d = d * (1 + rng.integers(0, 8, n) * 2.0**-52)
        else:
            d = _logu(rng, 1e-16, 1e6, n)
        per_cell = np.min(A / d)
        once = A / np.max(d)
        assert per_cell.tobytes() == np.float64(once).tobytes()


def test_min_of_divergence_term_is_term_of_min():
    # dtdivt: per cell (w/2vol < -g_small) ? s * RN(-1 / RN(w/2vol)) : g_big
    rng = np.random.default_rng(12)
    g_small, g_big, s = 1.0e-16, 1.0e21, 0.7
    for _ in range(200):
        vol2 = 2.0 * float(_logu(rng, 1e-8, 1.0, 1)[0])
        n = int(rng.integers(1, 64))
        w = rng.normal(0.0, 1.0, n) * float(_logu(rng, 1e-20, 1.0, 1)[0])
        dvv = w / vol2
        cell = np.where(dvv < -g_small, s * (-1.0 / np.where(dvv < -g_small, dvv, -1.0)), g_big)
        m = np.min(w) / vol2
        once = s * (-1.0 / m) if m < -g_small else g_big
        assert np.float64(np.min(cell)).tobytes() == np.float64(once).tobytes()


def test_max_of_rounded_sqrt_is_sqrt_of_max():
    # DtAcc: max_i fmax(RN(sqrt(a_i)), g) == fmax(RN(sqrt(max_i a_i)), g)
    rng = np.random.default_rng(13)
    g = 1.0e-16
    for trial in range(300):
        n = int(rng.integers(1, 64))
        if trial % 3 == 0:  # near-ties in the last ulps
            a = np.full(n, float(_logu(rng, 1e-40, 1e6, 1)[0]))
            a = a * (1 + rng.integers(0, 8, n) * 2.0**-52)
        else:
            a = _logu(rng, 1e-40, 1e6, n)
        if trial % 5 == 0:
            a[rng.integers(0, n)] = 0.0
        per_cell = np.max(np.fmax(np.sqrt(a), g))
        once = np.fmax(np.sqrt(np.max(a)), g)
        assert np.float64(per_cell).tobytes() == np.float64(once).tobytes()


def test_max_of_rounded_square_of_sqrt_is_that_of_max():
    # DtAcc: cells with q = 0 contribute cc2 = RN(RN(sqrt(c2))^2), a monotone
    # function of c2, so max_i f(c2_i) == f(max_i c2_i); cells with q != 0
    # keep their own cc2 and the two maxima combine exactly.
    rng = np.random.default_rng(14)
    for trial in range(300):
        n = int(rng.integers(1, 64))
        if trial % 3 == 0:  # near-ties in the last ulps
            c2 = np.full(n, float(_logu(rng, 1e-30, 1e4, 1)[0]))
            c2 = c2 * (1 + rng.integers(0, 16, n) * 2.0**-52)
        else:
            c2 = _logu(rng, 1e-30, 1e4, n)
        q = np.where(rng.uniform(size=n) < 0.3, _logu(rng, 1e-12, 1.0, n), 0.0)
        rho = _logu(rng, 1e-2, 1e2, n)
        cs = np.sqrt(c2)
        per_cell = np.max(cs * cs + 2.0 * q / rho)
        z = q == 0.0
        m1 = np.max(c2[z]) if z.any() else 0.0
        s1 = np.sqrt(m1)
        m2 = np.max((cs * cs + 2.0 * q / rho)[~z]) if (~z).any() else 0.0
        once = max(s1 * s1, m2)
        assert np.float64(per_cell).tobytes() == np.float64(once).tobytes()
