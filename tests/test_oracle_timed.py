"""The timed oracle mode (the CPU baseline of BASELINE.md §4: OpenMP at the paper's chunk sizes,
fp64 Makhoul FFT transforms) against the plain oracle it speeds up, CPU only.  The FFT
transforms are also checked against scipy.fft (DCT-II / DCT-III / DST-III)."""
import numpy as np
import pytest
import scipy.fft

import oracle
from synth import make_netlist, make_positions


@pytest.mark.parametrize("n", [2, 8, 64, 512])
@pytest.mark.parametrize("kind", [oracle.DCT, oracle.IDCT, oracle.IDXST])
def test_fft_transforms_equal_naive(n, kind):
    a = np.random.default_rng(n + 10 * kind).standard_normal((5, n))
    naive = oracle.transform(kind, a, 1)
    fast = oracle.transform_fft(kind, a, 1, 4)
    np.testing.assert_allclose(fast, naive, rtol=0, atol=1e-12 * max(1.0, np.abs(naive).max()))


def test_fft_transforms_against_scipy():
    a = np.random.default_rng(7).standard_normal((3, 256))
    n = a.shape[1]
    # eq (7a) x 2/n = scipy DCT-II / n; eq (7b) = scipy DCT-III / 2; eq (8a) = DST-III of x_1.. / 2
    np.testing.assert_allclose(oracle.transform_fft(oracle.DCT, a, 1, 2), scipy.fft.dct(a, 2) / n, atol=1e-12)
    np.testing.assert_allclose(oracle.transform_fft(oracle.IDCT, a, 1, 2), scipy.fft.dct(a, 3) / 2, atol=1e-12)
    b = np.concatenate([a[:, 1:], np.zeros((3, 1))], axis=1)   # x_1 .. x_{n-1}, x_n = 0
    np.testing.assert_allclose(oracle.transform_fft(oracle.IDXST, a, 1, 2), scipy.fft.dst(b, 3) / 2, atol=1e-12)


@pytest.mark.parametrize("threads", [1, 3])
def test_evaluate_timed_equals_evaluate(threads):
    nl = make_netlist("tiny")
    for dist in ("spread", "initial"):
        x, y = make_positions(nl, dist)
        ref = oracle.evaluate(nl, x, y, nl.bin_w, 0.7, with_hpwl=False)
        got = oracle.evaluate_timed(nl, x, y, nl.bin_w, 0.7, threads)
        for k in ("obj", "wl", "energy"):
            assert got[k] == pytest.approx(ref[k], rel=1e-11), k
        for k in ("gx", "gy"):
            np.testing.assert_allclose(got[k], ref[k], rtol=1e-9, atol=1e-11 * np.abs(ref[k]).max())
