"""Pins for the oracle's LSE wirelength and its gradient (CPU only).

PAPER.md names log-sum-exp wirelength as "also implemented" without printing it;
reading A27 takes the definition of its reference [29]:
    LSE_e = gamma ln sum_i e^{x_i/gamma} + gamma ln sum_i e^{-x_i/gamma}   (per axis).
Each test checks the oracle against something other than itself: a closed form derived by
hand, bounds that follow from the definition, 50-digit evaluation of the unshifted formula,
finite differences, or an invariant.
"""
import math

import mpmath
import numpy as np
import pytest

import oracle
from synth import custom_netlist, make_netlist, make_positions


def _two_pin(d):
    nl = custom_netlist([0, 2], [0, 1], [0, 0], [0, 0], [1, 1], [1, 1], (0, 0, 1e6, 1e6), (64, 64))
    x = np.array([100.0, 100.0 + d], dtype=np.float32)
    y = np.array([50.0, 50.0], dtype=np.float32)
    return nl, x, y


@pytest.mark.parametrize("d,gamma", [(1.0, 0.5), (8.0, 4.0), (3.0, 30.0), (64.0, 2.0), (0.25, 1.0)])
def test_two_pin_closed_form(d, gamma):
    """Two pins at separation d: gamma ln(e^{a/g} + e^{b/g}) = max + gamma ln(1 + e^{-d/g}) on each
    side, so LSE_x = d + 2 gamma ln(1 + e^{-d/gamma}); the y axis (coincident) gives 2 gamma ln 2.
    dLSE/dx_2 = 1/(1 + e^{-t}) - e^{-t}/(1 + e^{-t}) = tanh(t/2), t = d/gamma."""
    nl, x, y = _two_pin(d)
    wl, gx, gy = oracle.lse(nl, x, y, gamma)
    t = d / gamma
    assert wl == pytest.approx(d + 2 * gamma * math.log1p(math.exp(-t)) + 2 * gamma * math.log(2),
                               rel=1e-12)
    assert gx[1] == pytest.approx(math.tanh(t / 2), rel=1e-9, abs=1e-15)
    assert gx[0] == pytest.approx(-math.tanh(t / 2), rel=1e-9, abs=1e-15)
    assert abs(gy[0]) < 1e-15 and abs(gy[1]) < 1e-15


def _random_nets(rng, n_nets, dmax, spread):
    deg = rng.integers(2, dmax + 1, size=n_nets)
    ns = np.concatenate([[0], np.cumsum(deg)])
    npins = int(ns[-1])
    nl = custom_netlist(ns, np.arange(npins), np.zeros(npins), np.zeros(npins),
                        np.ones(npins), np.ones(npins), (0, 0, 1e6, 1e6), (64, 64))
    x = (1000 + rng.random(npins) * spread).astype(np.float32)
    y = (2000 + rng.random(npins) * spread).astype(np.float32)
    return nl, x, y


def test_lse_bounds_vs_hpwl():
    """max_i x_i <= gamma ln sum e^{x_i/gamma} <= max_i x_i + gamma ln d, hence per net
    0 <= LSE_e - HPWL_e <= 2 gamma ln d per axis (4 gamma ln d for x + y)."""
    rng = np.random.default_rng(15)
    nl, x, y = _random_nets(rng, 400, 12, 300.0)
    d = nl.degrees()
    h = oracle.hpwl_nets(nl, x, y)
    for gamma in (0.3, 3.0, 30.0):
        _, _, _, wl = oracle.lse(nl, x, y, gamma, per_net=True)
        gap = wl - h
        assert np.all(gap >= -1e-9)
        assert np.all(gap <= 4 * gamma * np.log(d) + 1e-9)


def test_coincident_pins():
    """All d pins at one point: each log-sum is x + gamma ln d, so LSE = 2 gamma ln d per axis and
    the gradient is (1/d - 1/d) = 0 for every pin; degree-1 nets give 0 (reading A3)."""
    nl = custom_netlist([0, 3, 4], [0, 0, 0, 1], [1, 1, 1, 0], [2, 2, 2, 0], [4, 4], [4, 4],
                        (0, 0, 1e4, 1e4), (16, 16))
    x = np.array([500.0, 900.0], dtype=np.float32)
    y = np.array([700.0, 100.0], dtype=np.float32)
    gamma = 3.0
    wl, gx, gy = oracle.lse(nl, x, y, gamma)
    assert wl == pytest.approx(4 * gamma * math.log(3), rel=1e-14)
    assert np.all(np.abs(gx) < 1e-14) and np.all(np.abs(gy) < 1e-14)
    assert gx[1] == 0.0 and gy[1] == 0.0


def test_lse_tends_to_hpwl():
    rng = np.random.default_rng(16)
    nl, x, y = _random_nets(rng, 100, 8, 500.0)
    h = oracle.hpwl(nl, x, y)
    errs = [abs(oracle.lse(nl, x, y, g)[0] - h) / h for g in (10.0, 1.0, 0.1, 0.01)]
    assert errs[-1] < 1e-4
    assert all(errs[i + 1] < errs[i] for i in range(3))


def test_lse_matches_unshifted_definition_in_50_digits():
    """The shift is an equivalent transformation: the literal definition of [29] without
    the shift, evaluated with 50-digit arithmetic, equals the oracle."""
    rng = np.random.default_rng(17)
    nl, x, y = _random_nets(rng, 30, 9, 80.0)
    gamma = 2.5
    _, _, _, wl = oracle.lse(nl, x, y, gamma, per_net=True)
    mpmath.mp.dps = 50
    for e in range(nl.num_nets):
        s, t = nl.net_start[e], nl.net_start[e + 1]
        tot = mpmath.mpf(0)
        for coords in (x[nl.pin2cell[s:t]], y[nl.pin2cell[s:t]]):
            xs = [mpmath.mpf(float(v)) for v in coords]
            tot += gamma * mpmath.log(sum(mpmath.exp(v / gamma) for v in xs))
            tot += gamma * mpmath.log(sum(mpmath.exp(-v / gamma) for v in xs))
        assert float(tot) == pytest.approx(wl[e], rel=1e-12)


def test_lse_gradient_finite_difference():
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    nl.net_weight = np.random.default_rng(13).uniform(0.5, 2.0, nl.num_nets).astype(np.float32)
    gamma = 4.0 * nl.bin_w
    _, gx, gy = oracle.lse(nl, x, y, gamma)
    rng = np.random.default_rng(14)
    xs = x.astype(np.float64)
    ys = y.astype(np.float64)
    h = 1e-4
    for c in rng.choice(nl.num_cells, 25, replace=False):
        for axis, g in ((0, gx), (1, gy)):
            a = xs.copy() if axis == 0 else ys.copy()
            a[c] += h
            fp = oracle.lse(nl, a if axis == 0 else xs, ys if axis == 0 else a, gamma)[0]
            a[c] -= 2 * h
            fm = oracle.lse(nl, a if axis == 0 else xs, ys if axis == 0 else a, gamma)[0]
            assert g[c] == pytest.approx((fp - fm) / (2 * h), rel=1e-5, abs=1e-6)


def test_lse_invariants():
    """Translation: every net's pin gradients sum to zero (softmax minus softmax); each pin's
    gradient lies in [-1, 1] times the net weight; reflection x -> -x leaves LSE unchanged."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    gamma = 7.0
    wl, gx, gy = oracle.lse(nl, x, y, gamma)
    assert abs(gx.sum()) < 1e-9 * np.abs(gx).sum()
    assert abs(gy.sum()) < 1e-9 * np.abs(gy).sum()
    nl3 = make_netlist("tiny")
    nl3.pin_dx = -nl.pin_dx
    nl3.pin_dy = -nl.pin_dy
    wl3, gx3, _ = oracle.lse(nl3, -x, -y, gamma)
    assert wl3 == pytest.approx(wl, rel=1e-12)
    np.testing.assert_allclose(gx3, -gx, rtol=1e-9, atol=1e-12)
    rng = np.random.default_rng(18)
    nl4, x4, y4 = _random_nets(rng, 200, 10, 100.0)   # one cell per pin: pin gradients visible
    _, g4, _ = oracle.lse(nl4, x4, y4, 2.0)
    assert np.all(np.abs(g4) <= 1.0 + 1e-12)
