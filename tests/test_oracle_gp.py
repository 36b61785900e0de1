"""Pins for the GP-loop oracle (oracle/gp.py), CPU only.

What the paper fixes: the eq (18) density-weight factor and its stated behaviour over the
iterations.  What the mathematics fixes: Lipschitz step prediction on a quadratic
(the step is exactly 1/L, so an isotropic quadratic is minimised in one step), Nesterov
convergence on an ill-conditioned quadratic, the overflow of configurations with a known
density, the preconditioner's pin counts (brute force).  And one end-to-end property: from
the paper's initial placement the loop spreads the cells (overflow falls).
"""
import math

import numpy as np
import pytest

import oracle
from oracle import gp
from synth import custom_netlist, make_netlist, make_positions


def test_mu_follows_eq18_and_p452():
    """'from iteration 0 to 200, mu gradually drops from 1.05 to 1.03 and keeps this
    value afterward' (for p < 0); eq (18a): mu = mu_max at p = 0 (mu_max^(1-0)), 1 at p = 1,
    and never below mu_min."""
    prm = gp.GpParams()
    assert gp.mu(-1.0, 0, prm) == pytest.approx(1.05, abs=1e-15)
    m200 = gp.mu(-1.0, 200, prm)
    assert 1.029 <= m200 <= 1.031
    assert all(gp.mu(-0.5, k, prm) <= gp.mu(-0.5, k - 1, prm) for k in range(1, 400))
    assert gp.mu(-1.0, 203, prm) == gp.mu(-1.0, 5000, prm)     # "keeps this value afterward" (0.9999^k = 0.98 at k = 202)
    assert gp.mu(0.0, 10, prm) == pytest.approx(1.05, abs=1e-15)
    assert gp.mu(1.0, 10, prm) == pytest.approx(1.0, abs=1e-15)
    assert gp.mu(50.0, 10, prm) == 0.95


def test_lipschitz_step_solves_isotropic_quadratic_in_one_step():
    """f(z) = c/2 |z - z*|^2: ||dv|| / ||dg|| = 1/c exactly, so u_1 = v - g/c = z*."""
    rng = np.random.default_rng(0)
    c, zs = 3.7, rng.normal(size=50)
    v = rng.normal(size=50)
    vp = v + 1e-3 * rng.normal(size=50)
    grad = lambda z: c * (z - zs)  # noqa: E731
    u1, _, _, alpha = gp.nesterov_step(v.copy(), v, vp, grad(v), grad(vp), 1.0, 0.0, lambda z: z)
    assert alpha == pytest.approx(1 / c, rel=1e-12)
    np.testing.assert_allclose(u1, zs, rtol=0, atol=1e-12)


def test_nesterov_converges_on_ill_conditioned_quadratic():
    """Diagonal quadratic with condition number 100: the objective falls by > 1e6."""
    rng = np.random.default_rng(1)
    n = 200
    d = np.geomspace(1.0, 100.0, n)
    zs = rng.normal(size=n)
    f = lambda z: 0.5 * float(np.sum(d * (z - zs) ** 2))  # noqa: E731
    grad = lambda z: d * (z - zs)  # noqa: E731
    u = v = rng.normal(size=n)
    vp = v - 1e-3 * grad(v)
    g, gprev, a, alpha = grad(v), grad(vp), 1.0, 0.0
    f0 = f(u)
    for _ in range(300):
        u, vn, a, alpha = gp.nesterov_step(u, v, vp, g, gprev, a, alpha, lambda z: z)
        vp, gprev, v, g = v, g, vn, grad(vn)
    assert f(u) < 1e-6 * f0


def test_overflow_closed_forms():
    """One unstretched cell exactly covering one bin: rho = 1 there, so tau = (1 - t) b^2 / (w h)
    = 1 - t; a uniform tiling at density 1 has tau = 0 for t = 1."""
    b = 10.0
    nl = custom_netlist([0, 0], [], [], [], [b], [b], (0, 0, 16 * b, 16 * b), (16, 16))
    rho = oracle.density_map(nl, np.array([3 * b], np.float32), np.array([5 * b], np.float32), stretch=0)
    assert gp.overflow(nl, rho, 0.25) == pytest.approx(0.75, rel=1e-12)
    assert gp.overflow(nl, rho, 1.0) == 0.0
    n = 16
    xs, ys = np.meshgrid(np.arange(n) * b, np.arange(n) * b, indexing="ij")
    nl2 = custom_netlist([0, 0], [], [], [], np.full(n * n, b), np.full(n * n, b), (0, 0, n * b, n * b), (n, n))
    rho2 = oracle.density_map(nl2, xs.ravel().astype(np.float32), ys.ravel().astype(np.float32), stretch=0)
    assert gp.overflow(nl2, rho2, 1.0) == pytest.approx(0.0, abs=1e-12)
    assert gp.overflow(nl2, rho2, 0.5) == pytest.approx(0.5, rel=1e-12)


def test_gamma_schedule_endpoints():
    """A31 (RePlAce): gamma = 10 gamma_base at tau = 1 and gamma_base / 10 at tau = 0.1."""
    nl = make_netlist("tiny")
    prm = gp.GpParams()
    base = 4.0 * (nl.bin_w + nl.bin_h)
    assert gp.gamma_of(nl, 1.0, prm) == pytest.approx(10 * base, rel=1e-12)
    assert gp.gamma_of(nl, 0.1, prm) == pytest.approx(base / 10, rel=1e-12)


def test_cell_pins_brute_force():
    nl = make_netlist("tiny")
    nl.net_weight = np.random.default_rng(2).uniform(0.5, 2.0, nl.num_nets).astype(np.float32)
    ref = np.zeros(nl.num_cells)
    for e in range(nl.num_nets):
        for p in range(nl.net_start[e], nl.net_start[e + 1]):
            ref[nl.pin2cell[p]] += float(nl.net_weight[e])
    np.testing.assert_allclose(gp.cell_pins(nl), ref, rtol=1e-12)


def test_gp_loop_spreads_the_initial_placement():
    """From the paper's initial placement (cells at the centre with 0.1% noise) the
    loop spreads the cells: overflow falls well below its start, HPWL stays finite, lambda
    grows (the density term gains weight, eq 18)."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl, "initial")
    st = gp.gp_init(nl, x, y)
    tau0, lam0 = st.tau, st.lam
    hist = [gp.gp_step(nl, st) for _ in range(400)]
    assert tau0 > 0.8
    assert hist[-1]["overflow"] < 0.1                  # DREAMPlace stops GP at 0.07-0.1
    assert min(h["overflow"] for h in hist[:100]) > 0.9 * tau0   # lambda_0 is small: WL first
    assert all(math.isfinite(h["hpwl"]) for h in hist)
    assert st.lam > lam0
    # cells stay inside the region (A33 clamp)
    assert np.all(st.u[0] >= nl.xl) and np.all(st.u[0] <= nl.xh - nl.cell_w + 1e-9)


def test_gp_stops_at_stop_overflow():
    """A36: once overflow < stop_overflow the loop is converged: positions, lambda and gamma no
    longer change (previously lambda grew by ~1.05 per iteration without bound)."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl, "initial")
    st = gp.gp_init(nl, x, y)
    hist = [gp.gp_step(nl, st) for _ in range(500)]
    k_stop = next(h["k"] for h in hist if h["overflow"] < 0.07)
    after = [h for h in hist if h["k"] > k_stop]
    assert len(after) > 10
    assert all(h["lam"] == after[0]["lam"] and h["gamma"] == after[0]["gamma"] for h in after)
    assert all(h["hpwl"] == after[0]["hpwl"] for h in after)
    u = st.u.copy()
    gp.gp_step(nl, st)
    assert np.array_equal(u, st.u)


def test_precondition_closed_form():
    """A29 on a hand-counted netlist: nets (c0, c1) weight 3 and (c0, c2) weight 0.5 give net-
    weighted pin counts P = (3.5, 3, 0.5); areas A = (8, 1, 0.25); at lambda = 0.25 the divisors
    max(1, P + lambda A) are (5.5, 3.25, 1) — the third clipped at 1."""
    nl = custom_netlist([0, 2, 4], [0, 1, 0, 2], [0.0] * 4, [0.0] * 4, [4.0, 1.0, 0.5], [2.0, 1.0, 0.5],
                        (0, 0, 160.0, 160.0), (16, 16), net_weight=[3.0, 0.5])
    gx = np.array([1.0, -2.0, 3.0])
    gy = np.array([-0.5, 0.25, 7.0])
    px, py = gp.precondition(nl, gx, gy, 0.25)
    d = np.array([5.5, 3.25, 1.0])
    np.testing.assert_allclose(px, gx / d, rtol=1e-15)
    np.testing.assert_allclose(py, gy / d, rtol=1e-15)
    # lambda = 0: the divisor is the pin count, never below 1
    px0, _ = gp.precondition(nl, gx, gy, 0.0)
    np.testing.assert_allclose(px0, gx / np.array([3.5, 3.0, 1.0]), rtol=1e-15)


def _two_cell_netlist():
    """Two 12 x 12 cells joined by one 2-pin net with pins at the cell centres (b = 10)."""
    return custom_netlist([0, 2], [0, 1], [6.0, 6.0], [6.0, 6.0], [12.0, 12.0], [12.0, 12.0],
                          (0, 0, 160.0, 160.0), (16, 16))


def test_gp_init_lambda0_against_closed_form_wa_gradient():
    """A32: lambda_0 = 8e-5 |grad WA|_1 / |grad D|_1 at the (clamped) start, gamma_0 = gamma(tau_0).
    |grad WA|_1 from the 2-pin closed form (dWA/dx_2 = sign(delta) [tanh(t/2) +
    (t/2) sech^2(t/2)], t = |delta| / gamma, per axis; the other pin the negative) — not from
    oracle.wa; |grad D|_1 from the density oracle (pinned by its own adjoint / mirror /
    convergence tests).  A wrong norm (L2), the WL value instead of its gradient, or a wrong
    scale fails this."""
    nl = _two_cell_netlist()
    x = np.array([30.0, 100.0], np.float32)
    y = np.array([40.0, 90.0], np.float32)
    st = gp.gp_init(nl, x, y)
    tau0 = gp.overflow(nl, oracle.density_map(nl, x, y), 1.0)
    gamma0 = gp.gamma_of(nl, tau0, gp.GpParams())
    assert st.tau == pytest.approx(tau0, rel=1e-12) and st.gamma == pytest.approx(gamma0, rel=1e-12)

    def pin_grad(delta):
        t = abs(delta) / gamma0
        return math.copysign(math.tanh(t / 2) + (t / 2) / math.cosh(t / 2) ** 2, delta)

    l1_wa = 2 * abs(pin_grad(70.0)) + 2 * abs(pin_grad(50.0))
    _, gdx, gdy, _ = oracle.density(nl, x, y, 1)
    l1_d = np.abs(gdx).sum() + np.abs(gdy).sum()
    assert st.lam == pytest.approx(8e-5 * l1_wa / l1_d, rel=1e-10)


def test_gp_init_first_lipschitz_point():
    """A33: v_{-1} = v_0 - eta g_0 with an rms displacement of exactly 0.01 b_x, along -g_0
    (g_0 = the preconditioned gradient at v_0, lambda_0); u_0 = v_0 = the clamped start."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl, "spread")
    x = x.astype(np.float64)
    x[0] = nl.xh + 50.0                       # outside: clamped to xh - w
    st = gp.gp_init(nl, x, y)
    assert st.v[0][0] == nl.xh - float(nl.cell_w[0])
    d = st.v - st.vp
    rms = math.sqrt(float(np.sum(d * d)) / d.size)
    assert rms == pytest.approx(0.01 * nl.bin_w, rel=1e-12)
    r = oracle.evaluate(nl, st.v[0], st.v[1], st.gamma, st.lam, with_hpwl=False)
    g0 = np.stack(gp.precondition(nl, r["gx"], r["gy"], st.lam))
    eta = float(np.sum(d * g0)) / float(np.sum(g0 * g0))
    assert eta > 0
    np.testing.assert_allclose(d, eta * g0, rtol=1e-12, atol=1e-12 * np.abs(d).max())
    assert np.array_equal(st.u, st.v) and st.a == 1.0 and st.k == 0


def test_overflow_with_fixed_macro_closed_form():
    """A30 with a fixed macro (A34): a macro exactly covering a 4 x 4 block of bins and nothing
    else overflows 0 at any target t (its charge counts at t), where the plain A30 would report
    16 (1 - t) bins of overflow; one movable unit cell on top of it overflows by its own area:
    tau = 1 (the movable area)."""
    b = 10.0
    nl = custom_netlist([0, 0], [], [], [], [4 * b, b], [4 * b, b], (0, 0, 16 * b, 16 * b), (16, 16))
    fixed = np.array([True, False])
    xm, ym = np.array([3 * b], np.float32), np.array([5 * b], np.float32)
    macro = custom_netlist([0, 0], [], [], [], [4 * b], [4 * b], (0, 0, 16 * b, 16 * b), (16, 16))
    rho_f = oracle.density_map(macro, xm, ym, stretch=0)
    for t in (0.7, 0.9, 1.0):
        assert gp.overflow(macro, rho_f, t) == pytest.approx(1.0 - t, abs=1e-12) or t == 1.0
        # macro alone, as a fixed cell: no overflow (movable area: the unit cell's)
        assert gp.overflow(nl, rho_f, t, fixed, rho_f) == pytest.approx(0.0, abs=1e-12)
        x = np.array([3 * b, 4 * b], np.float32)
        y = np.array([5 * b, 6 * b], np.float32)
        rho = oracle.density_map(nl, x, y, stretch=0)      # unit cell inside the macro's block
        assert gp.overflow(nl, rho, t, fixed, rho_f) == pytest.approx(1.0, rel=1e-12)
