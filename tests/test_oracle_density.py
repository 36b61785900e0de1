"""Pins for the oracle's density map, transforms, Poisson solve, energy and force gather.

PAPER.md: four-step decomposition P:251-256; density map P:310; force P:320-322;
eqs (4), (5) P:118-132, (7) P:324-331, (8) P:333-351, (9) P:353-365.
Readings A8-A22.  CPU only.
"""
import math

import numpy as np
import pytest
import scipy.fft

import oracle
from oracle import DCT, IDCT, IDXST
from synth import custom_netlist, make_netlist, make_positions


def _grid_nl(cells_w, cells_h, region, bins):
    n = len(cells_w)
    return custom_netlist([0], [], [], [], cells_w, cells_h, region, bins)


# ---------------------------------------------------------------------------- density map
def test_area_conservation():
    """sum rho b_x b_y = sum w h for cells whose (stretched) box lies inside (reading A9)."""
    nl = make_netlist("tiny")
    rng = np.random.default_rng(1)
    b = nl.bin_w
    W = nl.xh
    w = nl.cell_w.astype(np.float64)
    x = (2 * b + rng.random(nl.num_cells) * (W - w - 4 * b)).astype(np.float32)
    y = (2 * b + rng.random(nl.num_cells) * (W - 12 - 4 * b)).astype(np.float32)
    area = float(np.sum(nl.cell_w.astype(np.float64) * nl.cell_h))
    for stretch in (0, 1):
        rho = oracle.density_map(nl, x, y, stretch)
        assert rho.sum() * nl.bin_w * nl.bin_h == pytest.approx(area, rel=1e-12)


def test_cell_covering_one_bin():
    """A cell exactly covering one bin gives rho = 1 there and 0 elsewhere (stretch off)."""
    nl = _grid_nl([10.0], [10.0], (0, 0, 80, 80), (8, 8))
    rho = oracle.density_map(nl, np.array([30.0], np.float32), np.array([50.0], np.float32), 0)
    expect = np.zeros((8, 8))
    expect[3, 5] = 1.0
    np.testing.assert_array_equal(rho, expect)


def test_uniform_tiling_constant():
    """Cells tiling the region exactly give a constant map (= 1)."""
    m = 8
    xs, ys = np.meshgrid(np.arange(m) * 5.0, np.arange(m) * 5.0, indexing="ij")
    nl = _grid_nl(np.full(m * m, 5.0), np.full(m * m, 5.0), (0, 0, 40, 40), (m, m))
    rho = oracle.density_map(nl, xs.ravel().astype(np.float32), ys.ravel().astype(np.float32), 0)
    np.testing.assert_allclose(rho, 1.0, rtol=0, atol=1e-15)


def test_stretch_closed_form():
    """A small cell centred on a bin centre, stretched to sqrt2 b (reading A10): the centre
    bin holds r = w h / (2 b^2), edge neighbours r (sqrt2-1)/2, corners r ((sqrt2-1)/2)^2."""
    b = 10.0
    nl = _grid_nl([4.0], [6.0], (0, 0, 80, 80), (8, 8))
    x = np.array([45.0 - 2.0], np.float32)  # centre (45, 35) = centre of bin (4, 3)
    y = np.array([35.0 - 3.0], np.float32)
    rho = oracle.density_map(nl, x, y, 1)
    r = 4.0 * 6.0 / (2 * b * b)
    e = (math.sqrt(2) - 1) / 2
    assert rho[4, 3] == pytest.approx(r, rel=1e-12)
    for (i, j) in ((3, 3), (5, 3), (4, 2), (4, 4)):
        assert rho[i, j] == pytest.approx(r * e, rel=1e-12)
    for (i, j) in ((3, 2), (5, 4), (3, 4), (5, 2)):
        assert rho[i, j] == pytest.approx(r * e * e, rel=1e-12)
    assert rho.sum() == pytest.approx(4 * 6 / b / b, rel=1e-12)


# ------------------------------------------------------------------------------ transforms
@pytest.mark.parametrize("n", [8, 16, 64, 130])
def test_transforms_match_scipy(n):
    """eq 7a x 2/N == scipy DCT-II / N;  eq 7b == scipy DCT-III / 2;  eq 8a == scipy DST-III / 2
    applied to (x_1..x_{N-1}, 0)."""
    rng = np.random.default_rng(n)
    x = rng.standard_normal((3, n))
    np.testing.assert_allclose(oracle.transform(DCT, x, 1), scipy.fft.dct(x, type=2, axis=1) / n,
                               rtol=0, atol=1e-12)
    np.testing.assert_allclose(oracle.transform(IDCT, x, 1), scipy.fft.dct(x, type=3, axis=1) / 2,
                               rtol=0, atol=1e-12)
    z = np.concatenate([x[:, 1:], np.zeros((3, 1))], axis=1)
    np.testing.assert_allclose(oracle.transform(IDXST, x, 1), scipy.fft.dst(z, type=3, axis=1) / 2,
                               rtol=0, atol=1e-12)


def test_transform_closed_forms():
    n = 32
    c = 3.5
    out = oracle.transform(DCT, np.full((1, n), c), 1)[0]
    expect = np.zeros(n)
    expect[0] = 2 * c  # (2/N) N c
    np.testing.assert_allclose(out, expect, atol=1e-13)
    m = 5
    mode = np.cos(np.pi * m * (np.arange(n) + 0.5) / n)
    out = oracle.transform(DCT, mode[None], 1)[0]
    expect = np.zeros(n)
    expect[m] = 1.0  # (2/N)(N/2)
    np.testing.assert_allclose(out, expect, atol=1e-13)
    x = np.random.default_rng(0).standard_normal((2, n))
    np.testing.assert_allclose(oracle.transform(IDCT, oracle.transform(DCT, x, 1), 1), x, atol=1e-13)
    # eq (8e): IDXST(x)_k = (-1)^k IDCT({x_{N-n}})_k with x_N = 0
    rev = np.concatenate([np.zeros((2, 1)), x[:, :0:-1]], axis=1)
    sign = (-1.0) ** np.arange(n)
    np.testing.assert_allclose(oracle.transform(IDXST, x, 1), sign * oracle.transform(IDCT, rev, 1), atol=1e-12)


def test_dct2_is_eq5a_double_sum():
    """eq 9a (two 1-D passes) equals the double sum (2/M)^2 sum rho cos cos, brute force."""
    m = 8
    rho = np.random.default_rng(2).random((m, m))
    a = oracle.dct2(rho)
    t = np.arange(m) + 0.5
    for u in range(m):
        for v in range(m):
            s = sum(rho[i, j] * math.cos(math.pi * u * t[i] / m) * math.cos(math.pi * v * t[j] / m)
                    for i in range(m) for j in range(m))
            assert a[u, v] == pytest.approx(4 / m / m * s, abs=1e-13)


# -------------------------------------------------------------------------------- Poisson
def _smooth_density_nl(m, W=100.0):
    nl = _grid_nl([], [], (0, 0, W, W), (m, m))
    X = (np.arange(m) + 0.5) * (W / m)
    rho = np.exp(-((X[:, None] - 0.4 * W) ** 2 + (X[None, :] - 0.6 * W) ** 2) / (0.1 * W) ** 2)
    return nl, rho


def test_poisson_spectral_residual_and_zero_mean():
    nl, rho = _smooth_density_nl(32)
    a = oracle.dct2(rho)
    psi, xi_x, xi_y = oracle.fields(nl, a)
    ku, kv = oracle.wavenumbers(nl)
    k2 = ku[:, None] ** 2 + kv[None, :] ** 2
    ap = oracle.dct2(psi)
    mask = k2 > 0
    np.testing.assert_allclose((ap * k2)[mask], a[mask], rtol=0, atol=1e-12 * np.abs(a).max())
    assert abs(psi.mean()) < 1e-14 * np.abs(psi).max()   # eq 4c, reading A15


def test_single_mode_closed_form():
    """rho = cos(k_u X) cos(k_v Y) -> psi = rho / k^2, xi_X = (k_u/k^2) sin(k_u X) cos(k_v Y)."""
    m, W, H = 16, 64.0, 32.0
    nl = custom_netlist([0], [], [], [], [], [], (0, 0, W, H), (m, m))
    u, v = 3, 5
    X = (np.arange(m) + 0.5) * (W / m)
    Y = (np.arange(m) + 0.5) * (H / m)
    ku, kv = math.pi * u / W, math.pi * v / H
    rho = np.cos(ku * X)[:, None] * np.cos(kv * Y)[None, :]
    psi, xi_x, xi_y = oracle.fields(nl, oracle.dct2(rho))
    k2 = ku * ku + kv * kv
    np.testing.assert_allclose(psi, rho / k2, atol=1e-12)
    np.testing.assert_allclose(xi_x, ku / k2 * np.sin(ku * X)[:, None] * np.cos(kv * Y)[None, :], atol=1e-12)
    np.testing.assert_allclose(xi_y, kv / k2 * np.cos(ku * X)[:, None] * np.sin(kv * Y)[None, :], atol=1e-12)


def test_fd_laplacian_converges_second_order():
    """The 5-point Neumann finite-difference Laplacian of psi equals -(rho - mean rho) + O(b^2)
    (eq 4a/4b): the error falls ~4x per doubling of M."""
    errs = []
    for m in (32, 64, 128):
        nl, rho = _smooth_density_nl(m)
        psi, _, _ = oracle.fields(nl, oracle.dct2(rho))
        b = nl.bin_w
        p = np.pad(psi, 1, mode="edge")  # Neumann: mirror ghost cells
        lap = (p[2:, 1:-1] + p[:-2, 1:-1] + p[1:-1, 2:] + p[1:-1, :-2] - 4 * psi) / (b * b)
        errs.append(np.abs(lap + (rho - rho.mean())).max())
    assert 3.0 < errs[0] / errs[1] < 5.0 and 3.0 < errs[1] / errs[2] < 5.0


def test_energy_nonnegative_and_zero_for_uniform():
    m = 8
    xs, ys = np.meshgrid(np.arange(m) * 5.0, np.arange(m) * 5.0, indexing="ij")
    nl = _grid_nl(np.full(m * m, 5.0), np.full(m * m, 5.0), (0, 0, 40, 40), (m, m))
    D, gx, gy, _ = oracle.density(nl, xs.ravel().astype(np.float32), ys.ravel().astype(np.float32), 0)
    assert abs(D) < 1e-20 and np.abs(gx).max() < 1e-12 and np.abs(gy).max() < 1e-12
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    D, _, _, _ = oracle.density(nl, x, y, 1)
    assert D > 0


# ------------------------------------------------------------------------------- gather
def test_gather_adjoint_constant_field():
    """xi == 1 everywhere: gradient = -r sum ov = -w h for cells inside (reading A21)."""
    nl = make_netlist("tiny")
    rng = np.random.default_rng(8)
    b = nl.bin_w
    x = (2 * b + rng.random(nl.num_cells) * (nl.xh - 50 - 4 * b)).astype(np.float32)
    y = (2 * b + rng.random(nl.num_cells) * (nl.yh - 12 - 4 * b)).astype(np.float32)
    one = np.ones((nl.bins_x, nl.bins_y))
    gx, gy = oracle.density_grad(nl, x, y, one, 2 * one, 1)
    area = nl.cell_w.astype(np.float64) * nl.cell_h
    np.testing.assert_allclose(gx, -area, rtol=1e-12)
    np.testing.assert_allclose(gy, -2 * area, rtol=1e-12)


def test_centred_cell_feels_no_force_and_mirror_symmetry():
    nl = _grid_nl([20.0], [20.0], (0, 0, 160, 160), (16, 16))
    D, gx, gy, _ = oracle.density(nl, np.array([70.0], np.float32), np.array([70.0], np.float32), 1)
    assert abs(gx[0]) < 1e-9 and abs(gy[0]) < 1e-9
    # mirror x -> W - x - w: gx flips, gy and D unchanged
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    x = (np.round(x * 8) / 8).astype(np.float32)  # dyadic grid: the mirror below is exact
    D1, gx1, gy1, _ = oracle.density(nl, x, y, 1)
    xm = (nl.xh - x.astype(np.float64) - nl.cell_w).astype(np.float32)
    exact = np.abs(xm.astype(np.float64) - (nl.xh - x.astype(np.float64) - nl.cell_w)) == 0
    assert exact.all()
    D2, gx2, gy2, _ = oracle.density(nl, xm, y, 1)
    assert D2 == pytest.approx(D1, rel=1e-10)
    np.testing.assert_allclose(gx2, -gx1, rtol=1e-8, atol=1e-8 * np.abs(gx1).max())
    np.testing.assert_allclose(gy2, gy1, rtol=1e-8, atol=1e-8 * np.abs(gy1).max())


def test_force_converges_to_energy_derivative():
    """Reading A22: the paper's force gather is the continuum gradient of D, so its mismatch
    with the finite-difference derivative of the discrete D shrinks as bins refine."""
    rng = np.random.default_rng(9)
    n = 12
    W = 100.0
    w = rng.uniform(8, 16, n)
    h = rng.uniform(8, 16, n)
    x0 = rng.uniform(10, 70, n)
    y0 = rng.uniform(10, 70, n)
    rels = []
    for m in (16, 32, 64, 128):
        nl = _grid_nl(w, h, (0, 0, W, W), (m, m))
        nl.cell_w = w.astype(np.float32)
        nl.cell_h = h.astype(np.float32)
        x = x0.astype(np.float32)
        y = y0.astype(np.float32)
        _, gx, _, _ = oracle.density(nl, x, y, 0)
        fd = np.zeros(n)
        eps = 1e-3
        for i in range(n):
            xp = x.astype(np.float64).copy(); xp[i] += eps
            xm = x.astype(np.float64).copy(); xm[i] -= eps
            fd[i] = (oracle.density(nl, xp, y, 0)[0] - oracle.density(nl, xm, y, 0)[0]) / (2 * eps)
        rels.append(np.linalg.norm(gx - fd) / np.linalg.norm(fd))
    assert rels[-1] < 0.1
    assert rels[0] > rels[1] > rels[2] > rels[3]
