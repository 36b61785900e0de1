"""Plain fp64 CPU oracle for DREAMPlace's WA + electrostatic-density evaluation.

TEST INFRASTRUCTURE ONLY.  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this package.  It shares no code with the
CUDA path (paper_conf_dac_lindlrkp19_b200/) and never imports it; the only common
dependency is the seeded input generator in synth/.

The per-element loops live in dp_oracle.c (fp64, plain loops); this module converts the
fp32 inputs to fp64 exactly, composes the separable transforms exactly as eqs (9a)-(9d)
write them, and does the elementwise spectral scaling and the energy sum in numpy.

Citations "P:n" refer to /root/reference/PAPER.md line n; readings A1..A26 are listed in
DESIGN.md §3 (= SURVEY.md §8(c)).

Parity status: every function here is pinned by tests/test_oracle_*.py against closed
forms, invariants, library routines (scipy.fft.dct) or brute force.
The end-to-end scale of D against the paper is "parity unpinned": the paper prints no
value of D, psi, xi or any per-kernel quantity (last row).
"""
from __future__ import annotations

import ctypes
import math
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "dp_oracle.c")
_LIB_PATH = os.path.join(_HERE, "libdp_oracle.so")
_lib = None

DCT, IDCT, IDXST = 0, 1, 2


def build(force: bool = False) -> str:
    """Compile the C oracle with gcc (fp64, no fast-math, no FP contraction)."""
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < os.path.getmtime(_SRC):
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-fopenmp", "-ffp-contract=off", "-fno-fast-math",
                               "-shared", "-fPIC", "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB_PATH)
        P = ctypes.c_void_p
        I64, I32, D = ctypes.c_int64, ctypes.c_int, ctypes.c_double
        L.or_wa.restype = D
        L.or_wa.argtypes = [I64, P, P, P, P, P, P, P, D, P, P, P]
        L.or_lse.restype = D
        L.or_lse.argtypes = [I64, P, P, P, P, P, P, P, D, P, P, P]
        L.or_hpwl_nets.restype = None
        L.or_hpwl_nets.argtypes = [I64, P, P, P, P, P, P, P]
        L.or_density_map.restype = None
        L.or_density_map.argtypes = [I64, P, P, P, P, D, D, D, D, I32, I32, I32, P]
        L.or_density_grad.restype = None
        L.or_density_grad.argtypes = [I64, P, P, P, P, D, D, D, D, I32, I32, I32, P, P, P, P]
        L.or_transform_lastaxis.restype = None
        L.or_transform_lastaxis.argtypes = [I32, I64, I32, P, P]
        # timed mode (CPU baseline)
        L.or_wa_omp.restype = D
        L.or_wa_omp.argtypes = [I32, I64, P, P, P, P, P, P, P, D, P, P]
        L.or_density_map_omp.restype = None
        L.or_density_map_omp.argtypes = [I32, I64, P, P, P, P, D, D, D, D, I32, I32, I32, P]
        L.or_density_grad_omp.restype = None
        L.or_density_grad_omp.argtypes = [I32, I64, P, P, P, P, D, D, D, D, I32, I32, I32, P, P, P, P]
        L.or_transform_fft.restype = None
        L.or_transform_fft.argtypes = [I32, I32, I64, I32, P, P]
        _lib = L
    return _lib


def _p(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _f64(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.float64)


def _i32(a) -> np.ndarray:
    return np.ascontiguousarray(a, dtype=np.int32)


# --------------------------------------------------------------------------------------
# Wirelength
# --------------------------------------------------------------------------------------
def wa(nl, x, y, gamma: float, per_net: bool = False):
    """WA wirelength sum_e w_e (WL_e^x + WL_e^y) (eqs 2, 3, Table I)
    and its cell gradient (eq 6; reading A1).  Returns (total, gx, gy[, wl_net])."""
    ns, p2c = _i32(nl.net_start), _i32(nl.pin2cell)
    dx, dy = _f64(nl.pin_dx), _f64(nl.pin_dy)
    xx, yy = _f64(x), _f64(y)
    w = None if nl.net_weight is None else _f64(nl.net_weight)
    gx = np.zeros(nl.num_cells)
    gy = np.zeros(nl.num_cells)
    wl_net = np.zeros(nl.num_nets) if per_net else None
    tot = lib().or_wa(nl.num_nets, _p(ns), _p(p2c), _p(dx), _p(dy),
                      None if w is None else _p(w), _p(xx), _p(yy), float(gamma),
                      _p(gx), _p(gy), None if wl_net is None else _p(wl_net))
    return (tot, gx, gy, wl_net) if per_net else (tot, gx, gy)


def lse(nl, x, y, gamma: float, per_net: bool = False):
    """LSE wirelength sum_e w_e (LSE_e^x + LSE_e^y) (NEXT-3, reading A27: the
    definition of [29] with the P:159 shift) and its cell gradient.  Same returns as wa()."""
    ns, p2c = _i32(nl.net_start), _i32(nl.pin2cell)
    dx, dy = _f64(nl.pin_dx), _f64(nl.pin_dy)
    xx, yy = _f64(x), _f64(y)
    w = None if nl.net_weight is None else _f64(nl.net_weight)
    gx = np.zeros(nl.num_cells)
    gy = np.zeros(nl.num_cells)
    wl_net = np.zeros(nl.num_nets) if per_net else None
    tot = lib().or_lse(nl.num_nets, _p(ns), _p(p2c), _p(dx), _p(dy),
                       None if w is None else _p(w), _p(xx), _p(yy), float(gamma),
                       _p(gx), _p(gy), None if wl_net is None else _p(wl_net))
    return (tot, gx, gy, wl_net) if per_net else (tot, gx, gy)


def hpwl_nets(nl, x, y) -> np.ndarray:
    """Per-net HPWL h_e = (max px - min px) + (max py - min py) in fp64 (reading A6)."""
    h = np.zeros(nl.num_nets)
    lib().or_hpwl_nets(nl.num_nets, _p(_i32(nl.net_start)), _p(_i32(nl.pin2cell)),
                       _p(_f64(nl.pin_dx)), _p(_f64(nl.pin_dy)), _p(_f64(x)), _p(_f64(y)), _p(h))
    return h


def hpwl(nl, x, y) -> float:
    """Correctly rounded sum of the per-net HPWL values (reading A7: math.fsum is exact)."""
    return math.fsum(hpwl_nets(nl, x, y).tolist())


# --------------------------------------------------------------------------------------
# Density
# --------------------------------------------------------------------------------------
def density_map(nl, x, y, stretch: int = 1) -> np.ndarray:
    """rho[bins_x, bins_y] (readings A9, A10, A11, A20)."""
    rho = np.zeros((nl.bins_x, nl.bins_y))
    lib().or_density_map(nl.num_cells, _p(_f64(x)), _p(_f64(y)), _p(_f64(nl.cell_w)),
                         _p(_f64(nl.cell_h)), nl.xl, nl.yl, nl.xh, nl.yh,
                         nl.bins_x, nl.bins_y, int(stretch), _p(rho))
    return rho


def transform(kind: int, arr: np.ndarray, axis: int) -> np.ndarray:
    """Apply the naive 1-D DCT (eq 7a, x 2/N) / IDCT (eq 7b) / IDXST (eq 8a) along `axis`."""
    a = np.moveaxis(np.asarray(arr, dtype=np.float64), axis, -1)
    shape = a.shape
    src = np.ascontiguousarray(a.reshape(-1, shape[-1]))
    out = np.empty_like(src)
    lib().or_transform_lastaxis(int(kind), src.shape[0], src.shape[1], _p(src), _p(out))
    return np.moveaxis(out.reshape(shape), -1, axis)


def dct2(rho: np.ndarray) -> np.ndarray:
    """a_uv = DCT(DCT(rho)^T)^T  (eq 9a): the 1-D DCT of eq (7a) (x 2/N, reading A13)
    along y (rows), then along x.  Equals (2/Mx)(2/My) sum_xy rho cos(.) cos(.) of eq (5a)
    under reading A12/A13."""
    return transform(DCT, transform(DCT, rho, axis=1), axis=0)


def wavenumbers(nl):
    """Reading A12: k_u = pi u / W, k_v = pi v / H (physical wavenumbers of the cosine basis
    cos(pi u (x + 1/2) / M) of eq 7a on a region of width W)."""
    ku = np.pi * np.arange(nl.bins_x) / (nl.xh - nl.xl)
    kv = np.pi * np.arange(nl.bins_y) / (nl.yh - nl.yl)
    return ku, kv


def fields(nl, a: np.ndarray):
    """Potential and field from the spectrum (eqs 9b-9d; readings A12, A14, A15, A20):
        psi  = IDCT_x  IDCT_y  ( a / (ku^2 + kv^2) )
        xi_X = IDXST_x IDCT_y  ( a ku / (ku^2 + kv^2) )
        xi_Y = IDCT_x  IDXST_y ( a kv / (ku^2 + kv^2) )
    with the (0,0) term set to zero (eq 4c)."""
    ku, kv = wavenumbers(nl)
    k2 = ku[:, None] ** 2 + kv[None, :] ** 2
    inv = np.zeros_like(k2)
    nz = k2 > 0
    inv[nz] = 1.0 / k2[nz]
    a_psi = a * inv
    a_x = a * ku[:, None] * inv
    a_y = a * kv[None, :] * inv
    psi = transform(IDCT, transform(IDCT, a_psi, axis=1), axis=0)
    xi_x = transform(IDXST, transform(IDCT, a_x, axis=1), axis=0)
    xi_y = transform(IDCT, transform(IDXST, a_y, axis=1), axis=0)
    return psi, xi_x, xi_y


def energy(nl, rho: np.ndarray, psi: np.ndarray) -> float:
    """D = 1/2 b_x b_y sum_b rho_b psi_b  (reading A8: the potential energy of P:97 / P:256)."""
    return 0.5 * nl.bin_w * nl.bin_h * float(np.sum(rho * psi))


def density_grad(nl, x, y, xi_x, xi_y, stretch: int = 1):
    """dD/dx_i = -sum_b r_i ov(i,b) xi^X_b (reading A21)."""
    gx = np.zeros(nl.num_cells)
    gy = np.zeros(nl.num_cells)
    lib().or_density_grad(nl.num_cells, _p(_f64(x)), _p(_f64(y)), _p(_f64(nl.cell_w)),
                          _p(_f64(nl.cell_h)), nl.xl, nl.yl, nl.xh, nl.yh,
                          nl.bins_x, nl.bins_y, int(stretch),
                          _p(_f64(xi_x)), _p(_f64(xi_y)), _p(gx), _p(gy))
    return gx, gy


def density(nl, x, y, stretch: int = 1):
    """The four steps of P:251-256: rho -> a_uv -> (psi, xi) -> (D, dD/dx).
    Returns (D, gx, gy, parts) with parts = dict(rho, a, psi, xi_x, xi_y)."""
    rho = density_map(nl, x, y, stretch)
    a = dct2(rho)
    psi, xi_x, xi_y = fields(nl, a)
    D = energy(nl, rho, psi)
    gx, gy = density_grad(nl, x, y, xi_x, xi_y, stretch)
    return D, gx, gy, dict(rho=rho, a=a, psi=psi, xi_x=xi_x, xi_y=xi_y)


def region_blockage(nl, boxes, r: int) -> np.ndarray:
    """Reading A38 (fence regions): the blockage map of region r — the fraction of each
    bin outside the region, at density 1.  Fence r >= 1 is box r-1 (xl, yl, xh, yh); region 0,
    the default region, is the layout minus the (disjoint) fences.  Overlaps are the products
    of 1-D interval overlaps, as in the density map."""
    xs = nl.xl + np.arange(nl.bins_x + 1) * nl.bin_w
    ys = nl.yl + np.arange(nl.bins_y + 1) * nl.bin_h

    def cover(b):   # fraction of each bin inside box b
        ox = np.clip(np.minimum(xs[1:], b[2]) - np.maximum(xs[:-1], b[0]), 0.0, None) / nl.bin_w
        oy = np.clip(np.minimum(ys[1:], b[3]) - np.maximum(ys[:-1], b[1]), 0.0, None) / nl.bin_h
        return ox[:, None] * oy[None, :]

    if r == 0:
        out = np.zeros((nl.bins_x, nl.bins_y))
        for b in boxes:
            out += cover(b)
        return out
    return 1.0 - cover(boxes[r - 1])


def evaluate_regions(nl, x, y, gamma: float, lam: float, boxes, cell_region, stretch: int = 1):
    """Fence regions as "multiple electric fields, e.g., one for each region" (reading
    A38): region r has its own map rho_r = blockage_r + the charge of its cells, its own Poisson
    solve (eqs 9a-9d) and energy D_r; D = sum_r D_r, and a cell's density gradient is the force
    gather in its own region's field.  The wirelength part is unchanged (eq 2)."""
    cell_region = np.asarray(cell_region)
    wl, gwx, gwy = wa(nl, x, y, gamma)
    gdx = np.zeros(nl.num_cells)
    gdy = np.zeros(nl.num_cells)
    D = 0.0
    from synth import custom_netlist
    for r in range(len(boxes) + 1):
        idx = np.nonzero(cell_region == r)[0]
        sub = custom_netlist([0], [], [], [], nl.cell_w[idx], nl.cell_h[idx], (nl.xl, nl.yl, nl.xh, nl.yh),
                             (nl.bins_x, nl.bins_y))
        rho = region_blockage(nl, boxes, r) + density_map(sub, x[idx], y[idx], stretch)
        psi, xi_x, xi_y = fields(nl, dct2(rho))
        D += energy(nl, rho, psi)
        fx, fy = density_grad(sub, x[idx], y[idx], xi_x, xi_y, stretch)
        gdx[idx] = fx
        gdy[idx] = fy
    return dict(obj=wl + lam * D, wl=wl, energy=D, gx=gwx + lam * gdx, gy=gwy + lam * gdy, d_gx=gdx, d_gy=gdy)


def evaluate(nl, x, y, gamma: float, lam: float, stretch: int = 1, with_hpwl: bool = True,
             wl_model: str = "wa", fixed=None):
    """obj = WL + lambda D and grad = grad WL + lambda grad D (eq 2); WL = WA (eq 3)
    or LSE (reading A27).  fixed (bool [num_cells], NEXT-4 / reading A34): fixed cells
    are charges of the density (eq 1b's d(x, y) counts every cell) but not variables of
    (1a), so their gradient entries are 0."""
    wl, gwx, gwy = (lse if wl_model == "lse" else wa)(nl, x, y, gamma)
    D, gdx, gdy, parts = density(nl, x, y, stretch)
    if fixed is not None:
        m = np.asarray(fixed, dtype=bool)
        for g in (gwx, gwy, gdx, gdy):
            g[m] = 0.0
    out = dict(obj=wl + lam * D, wl=wl, energy=D, gx=gwx + lam * gdx, gy=gwy + lam * gdy,
               wl_gx=gwx, wl_gy=gwy, d_gx=gdx, d_gy=gdy, **parts)
    if with_hpwl:
        out["hpwl"] = hpwl(nl, x, y)
    return out


# --------------------------------------------------------------------------------------
# Timed mode: the CPU baseline of BASELINE.md §4 (never used for parity).  The same
# definitions with OpenMP over nets / cells at the paper's chunk sizes |E|/(T 16), |V|/(T 16)
# and fp64 Makhoul FFT transforms; validated against the plain functions
# above by tests/test_oracle_timed.py.
# --------------------------------------------------------------------------------------
def transform_fft(kind: int, arr: np.ndarray, axis: int, threads: int) -> np.ndarray:
    a = np.moveaxis(np.asarray(arr, dtype=np.float64), axis, -1)
    shape = a.shape
    src = np.ascontiguousarray(a.reshape(-1, shape[-1]))
    out = np.empty_like(src)
    lib().or_transform_fft(int(threads), int(kind), src.shape[0], src.shape[1], _p(src), _p(out))
    return np.moveaxis(out.reshape(shape), -1, axis)


def evaluate_timed(nl, x, y, gamma: float, lam: float, threads: int, stretch: int = 1):
    """obj = WA + lambda D and its gradient (eq 2) in the timed mode; returns the same keys as
    evaluate() minus the intermediate maps."""
    xd, yd = _f64(x), _f64(y)
    gwx = np.zeros(nl.num_cells)
    gwy = np.zeros(nl.num_cells)
    wl = lib().or_wa_omp(int(threads), nl.num_nets, _p(_i32(nl.net_start)), _p(_i32(nl.pin2cell)),
                         _p(_f64(nl.pin_dx)), _p(_f64(nl.pin_dy)),
                         None if nl.net_weight is None else _p(_f64(nl.net_weight)),
                         _p(xd), _p(yd), float(gamma), _p(gwx), _p(gwy))
    w, h = _f64(nl.cell_w), _f64(nl.cell_h)
    rho = np.zeros((nl.bins_x, nl.bins_y))
    lib().or_density_map_omp(int(threads), nl.num_cells, _p(xd), _p(yd), _p(w), _p(h), nl.xl, nl.yl, nl.xh,
                             nl.yh, nl.bins_x, nl.bins_y, int(stretch), _p(rho))
    a = transform_fft(DCT, transform_fft(DCT, rho, 1, threads), 0, threads)
    ku, kv = wavenumbers(nl)
    k2 = ku[:, None] ** 2 + kv[None, :] ** 2
    inv = np.zeros_like(k2)
    inv[k2 > 0] = 1.0 / k2[k2 > 0]
    psi = transform_fft(IDCT, transform_fft(IDCT, a * inv, 1, threads), 0, threads)
    xi_x = transform_fft(IDXST, transform_fft(IDCT, a * ku[:, None] * inv, 1, threads), 0, threads)
    xi_y = transform_fft(IDCT, transform_fft(IDXST, a * kv[None, :] * inv, 1, threads), 0, threads)
    D = energy(nl, rho, psi)
    gdx = np.empty(nl.num_cells)
    gdy = np.empty(nl.num_cells)
    lib().or_density_grad_omp(int(threads), nl.num_cells, _p(xd), _p(yd), _p(w), _p(h), nl.xl, nl.yl, nl.xh,
                              nl.yh, nl.bins_x, nl.bins_y, int(stretch), _p(np.ascontiguousarray(xi_x)),
                              _p(np.ascontiguousarray(xi_y)), _p(gdx), _p(gdy))
    return dict(obj=wl + lam * D, wl=wl, energy=D, gx=gwx + lam * gdx, gy=gwy + lam * gdy)
