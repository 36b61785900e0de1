"""Pins for the oracle's WA wirelength, its gradient and HPWL (CPU only).

Each test checks the oracle against something other than itself: a closed form, a bound
derived from eq (3), brute force in arbitrary precision, finite differences, or an
invariant.  PAPER.md: eq (3), Table I, shift P:159, eq (6) P:161.
"""
import math
from fractions import Fraction

import mpmath
import numpy as np
import pytest

import oracle
from synth import custom_netlist, make_netlist, make_positions


def _two_pin(d, gamma, dy=0.0):
    nl = custom_netlist([0, 2], [0, 1], [0, 0], [0, 0], [1, 1], [1, 1], (0, 0, 1e6, 1e6), (64, 64))
    x = np.array([100.0, 100.0 + d], dtype=np.float32)
    y = np.array([50.0, 50.0 + dy], dtype=np.float32)
    return nl, x, y


@pytest.mark.parametrize("d,gamma", [(1.0, 0.5), (8.0, 4.0), (3.0, 30.0), (64.0, 2.0), (0.25, 1.0)])
def test_two_pin_closed_form(d, gamma):
    """2-pin net at separation d: WA = d tanh(d/(2 gamma)); dWA/dx_2 = tanh(t/2) + (t/2) sech^2(t/2)."""
    nl, x, y = _two_pin(d, gamma)
    d = float(x[1]) - float(x[0])
    wl, gx, gy = oracle.wa(nl, x, y, gamma)
    t = d / gamma
    assert wl == pytest.approx(d * math.tanh(t / 2), rel=1e-12, abs=1e-12)
    g = math.tanh(t / 2) + (t / 2) / math.cosh(t / 2) ** 2
    assert gx[1] == pytest.approx(g, rel=1e-9, abs=1e-12)
    assert gx[0] == pytest.approx(-g, rel=1e-9, abs=1e-12)
    assert gy[0] == pytest.approx(0.0, abs=1e-9) and gy[1] == pytest.approx(0.0, abs=1e-9)


def test_degenerate_nets():
    """Coincident pins -> WA = 0 and gradient 0; degree-1 and degree-0 nets -> 0 (reading A3)."""
    nl = custom_netlist([0, 3, 4, 4], [0, 0, 0, 1], [1, 1, 1, 0], [2, 2, 2, 0], [4, 4], [4, 4],
                        (0, 0, 1e4, 1e4), (16, 16))
    x = np.array([500.0, 900.0], dtype=np.float32)
    y = np.array([700.0, 100.0], dtype=np.float32)
    wl, gx, gy = oracle.wa(nl, x, y, 3.0)
    assert abs(wl) < 1e-9
    assert np.all(np.abs(gx) < 1e-9) and np.all(np.abs(gy) < 1e-9)
    assert gx[1] == 0.0 and gy[1] == 0.0  # the degree-1 net's cell gets exactly nothing


def _random_nets(rng, n_nets, dmax, spread):
    deg = rng.integers(2, dmax + 1, size=n_nets)
    ns = np.concatenate([[0], np.cumsum(deg)])
    npins = int(ns[-1])
    nc = npins  # one cell per pin: positions are then free per pin
    nl = custom_netlist(ns, np.arange(npins), np.zeros(npins), np.zeros(npins),
                        np.ones(nc), np.ones(nc), (0, 0, 1e6, 1e6), (64, 64))
    x = (1000 + rng.random(nc) * spread).astype(np.float32)
    y = (2000 + rng.random(nc) * spread).astype(np.float32)
    return nl, x, y


def test_wa_bounds_vs_hpwl():
    """0 <= HPWL_e - WA_e <= 2 (d-1) gamma / e per axis (derived from eq 3: each weighted mean
    lies in [x-, x+] and is within (d-1) max_s s e^{-s/gamma} = (d-1) gamma/e of its extreme)."""
    rng = np.random.default_rng(5)
    nl, x, y = _random_nets(rng, 400, 12, 300.0)
    for gamma in (0.3, 3.0, 30.0):
        _, _, _, wl = oracle.wa(nl, x, y, gamma, per_net=True)
        h = oracle.hpwl_nets(nl, x, y)
        d = nl.degrees()
        gap = h - wl
        assert np.all(gap >= -1e-9)
        assert np.all(gap <= 2 * 2 * (d - 1) * gamma / math.e + 1e-9)  # x + y


def test_wa_tends_to_hpwl():
    """WA -> HPWL as gamma -> 0."""
    rng = np.random.default_rng(6)
    nl, x, y = _random_nets(rng, 100, 8, 500.0)
    h = oracle.hpwl(nl, x, y)
    errs = [abs(oracle.wa(nl, x, y, g)[0] - h) / h for g in (10.0, 1.0, 0.1, 0.01)]
    assert errs[-1] < 1e-4
    assert all(errs[i + 1] < errs[i] for i in range(3))


def test_wa_matches_unshifted_eq3_in_50_digits():
    """The shift of P:159 is an equivalent transformation: literal eq (3) (no shift) evaluated
    with 50-digit arithmetic equals the oracle."""
    rng = np.random.default_rng(7)
    nl, x, y = _random_nets(rng, 30, 9, 80.0)
    gamma = 2.5
    _, _, _, wl = oracle.wa(nl, x, y, gamma, per_net=True)
    mpmath.mp.dps = 50
    for e in range(nl.num_nets):
        s, t = nl.net_start[e], nl.net_start[e + 1]
        tot = mpmath.mpf(0)
        for coords in (x[nl.pin2cell[s:t]], y[nl.pin2cell[s:t]]):
            xs = [mpmath.mpf(float(v)) for v in coords]
            ep = [mpmath.exp(v / gamma) for v in xs]
            em = [mpmath.exp(-v / gamma) for v in xs]
            tot += sum(v * a for v, a in zip(xs, ep)) / sum(ep) - sum(v * a for v, a in zip(xs, em)) / sum(em)
        assert float(tot) == pytest.approx(wl[e], rel=1e-12)


def test_wa_gradient_finite_difference():
    """Central finite differences of the oracle's own WA value in fp64 (reading A1: cell
    coordinates, pin offsets, shared cells, net weights)."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    nl.net_weight = np.random.default_rng(3).uniform(0.5, 2.0, nl.num_nets).astype(np.float32)
    gamma = 4.0 * nl.bin_w
    _, gx, gy = oracle.wa(nl, x, y, gamma)
    rng = np.random.default_rng(4)
    xs = x.astype(np.float64)
    ys = y.astype(np.float64)
    h = 1e-4
    for c in rng.choice(nl.num_cells, 25, replace=False):
        for axis, g in ((0, gx), (1, gy)):
            a = xs.copy() if axis == 0 else ys.copy()
            a[c] += h
            fp = oracle.wa(nl, a if axis == 0 else xs, ys if axis == 0 else a, gamma)[0]
            a[c] -= 2 * h
            fm = oracle.wa(nl, a if axis == 0 else xs, ys if axis == 0 else a, gamma)[0]
            fd = (fp - fm) / (2 * h)
            assert g[c] == pytest.approx(fd, rel=1e-5, abs=1e-6)


def test_wa_invariants():
    """Translation: the gradient of every net sums to zero, so the total over cells does;
    scaling: WA(s x; s gamma) = s WA(x; gamma); reflection x -> -x leaves WA unchanged."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    gamma = 7.0
    wl, gx, gy = oracle.wa(nl, x, y, gamma)
    assert abs(gx.sum()) < 1e-9 * np.abs(gx).sum()
    assert abs(gy.sum()) < 1e-9 * np.abs(gy).sum()
    # scaling by a power of two keeps the fp32 inputs exact; pin offsets scale too
    nl2 = make_netlist("tiny")
    nl2.pin_dx = nl.pin_dx * 4
    nl2.pin_dy = nl.pin_dy * 4
    wl2, _, _ = oracle.wa(nl2, x * 4, y * 4, gamma * 4)
    assert wl2 == pytest.approx(4 * wl, rel=1e-12)
    nl3 = make_netlist("tiny")
    nl3.pin_dx = -nl.pin_dx
    nl3.pin_dy = -nl.pin_dy
    wl3, gx3, gy3 = oracle.wa(nl3, -x, -y, gamma)
    assert wl3 == pytest.approx(wl, rel=1e-12)
    np.testing.assert_allclose(gx3, -gx, rtol=1e-9, atol=1e-12)


def test_hpwl_brute_force_and_exact_sum():
    """HPWL (reading A6) by brute force over pins with exact rational summation."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    px = x.astype(np.float64)[nl.pin2cell] + nl.pin_dx.astype(np.float64)
    py = y.astype(np.float64)[nl.pin2cell] + nl.pin_dy.astype(np.float64)
    exact = Fraction(0)
    for e in range(nl.num_nets):
        s, t = nl.net_start[e], nl.net_start[e + 1]
        if t - s < 2:
            continue
        he = (max(px[s:t]) - min(px[s:t])) + (max(py[s:t]) - min(py[s:t]))
        exact += Fraction(he)
    assert oracle.hpwl(nl, x, y) == float(exact)  # correctly rounded (Fraction -> float rounds once)


def test_net_weight_scales():
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    wl, gx, _ = oracle.wa(nl, x, y, 5.0)
    nl.net_weight = np.full(nl.num_nets, 2.0, dtype=np.float32)
    wl2, gx2, _ = oracle.wa(nl, x, y, 5.0)
    assert wl2 == pytest.approx(2 * wl, rel=1e-14)
    np.testing.assert_allclose(gx2, 2 * gx, rtol=1e-14, atol=0)
