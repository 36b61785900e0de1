"""Plain fp64 oracle of the global-placement loop around the evaluation.

TEST INFRASTRUCTURE ONLY (same rules as oracle/__init__.py: imported by tests/, smoke() and
bench.py's CPU legs only; shares no code with the CUDA path).

PAPER.md describes the loop only in outline: "the kernel GP iterations refer to the loop that
involves the computation of wirelength and density gradient, optimization engines, and cell
location updating"; the optimizer is "Nesterov's method as the gradient-descent
solver with a Lipschitz-constant approximation scheme for line search" of ePlace/RePlAce
[6], [8]; the density weight follows eq (18) with the DREAMPlace modification
(P:441-452).  Everything the paper does not print is taken from the ePlace/RePlAce
conventions the paper says it follows and listed as readings in DESIGN.md §3:

  A28  Nesterov with Lipschitz step prediction (ePlace [6]), no backtracking:
         alpha_k = ||v_k - v_{k-1}||_2 / ||g_k - g_{k-1}||_2   (g = preconditioned gradient)
         u_{k+1} = clamp(v_k - alpha_k g_k)
         a_{k+1} = (1 + sqrt(4 a_k^2 + 1)) / 2
         v_{k+1} = clamp(u_{k+1} + (a_k - 1)/a_{k+1} (u_{k+1} - u_k))
       alpha_k keeps its previous value if ||g_k - g_{k-1}|| = 0.
  A29  preconditioner (ePlace): g_i = grad_i / max(1, P_i + lambda A_i), P_i = pins of cell i
       (net-weighted), A_i = w_i h_i.
  A30  overflow tau = sum_b max(rho_b - t, 0) b_x b_y / sum_i w_i h_i on the evaluation's own
       (stretched, reading A10) bin map; target density t (default 1.0).
  A31  gamma schedule (RePlAce): gamma = gamma_base 10^((tau - 0.1) 20/9 - 1), gamma_base =
       4 (b_x + b_y).
  A32  lambda_0 = s ||grad WA||_1 / ||grad D||_1 at the start point (s = 8e-5), then eq (18)
       every iteration with p = (HPWL_{k+1} - HPWL_k) / 3.5e5 and, for p < 0,
       mu = mu_max max(0.9999^k, 0.98).
  A33  HPWL and tau are taken at the reference solution v, where the gradient is evaluated;
       clamp keeps lower-left corners in [xl, xh - w] x [yl, yh - h]; the first Lipschitz
       estimate uses v_{-1} = v_0 - eta g_0 with an rms displacement of 0.01 b_x.
  A36  GP stops once tau < stop_overflow (DREAMPlace's stop criterion, default 0.07): later
       iterations leave u, v, lambda and gamma unchanged ("GP converges"); lambda is
       capped at 1e30 (the eq-18 product is unbounded otherwise).
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

from . import density_map, evaluate


@dataclasses.dataclass
class GpParams:
    target_density: float = 1.0
    gamma_base_scale: float = 4.0     # gamma_base = scale (b_x + b_y)          (A31)
    lambda_scale: float = 8e-5        # lambda_0 = scale |grad WA|_1/|grad D|_1  (A32)
    mu_min: float = 0.95              # eq (18a)
    mu_max: float = 1.05
    dhpwl_ref: float = 3.5e5          # p = dHPWL / 3.5e5
    init_rms_bins: float = 0.01       # rms displacement of v_{-1}, in bins      (A33)
    stop_overflow: float = 0.07       # GP converged below this overflow         (A36)


# ------------------------------------------------------------------------- schedule pieces
def mu(p: float, k: int, prm: GpParams) -> float:
    """eq (18a) with the DREAMPlace change for p < 0."""
    if p < 0:
        return prm.mu_max * max(0.9999 ** k, 0.98)
    return max(prm.mu_min, prm.mu_max ** (1.0 - p))


def overflow(nl, rho: np.ndarray, target: float, fixed=None, rho_fixed=None) -> float:
    """A30: sum_b max(rho_b - t, 0) b_x b_y / total cell area.  With fixed cells (A34; the
    DREAMPlace convention): the fixed charge counts at the target density, rho_eff = rho_movable
    + t rho_fixed = rho - (1 - t) rho_fixed, and the sum is divided by the movable area."""
    a = nl.cell_w.astype(np.float64) * nl.cell_h.astype(np.float64)
    if fixed is not None:
        a = a[~np.asarray(fixed, dtype=bool)]
        rho = rho - (1.0 - target) * rho_fixed
    return float(np.sum(np.maximum(rho - target, 0.0))) * nl.bin_w * nl.bin_h / float(np.sum(a))


def gamma_of(nl, tau: float, prm: GpParams) -> float:
    """A31 (RePlAce): gamma_base 10^((tau - 0.1) 20/9 - 1)."""
    base = prm.gamma_base_scale * (nl.bin_w + nl.bin_h)
    return base * 10.0 ** ((tau - 0.1) * 20.0 / 9.0 - 1.0)


def cell_pins(nl) -> np.ndarray:
    """P_i of A29: net-weighted pin count of each cell."""
    w = np.ones(nl.num_nets) if nl.net_weight is None else nl.net_weight.astype(np.float64)
    per_pin = np.repeat(w, np.diff(nl.net_start))
    return np.bincount(nl.pin2cell, weights=per_pin, minlength=nl.num_cells)


def precondition(nl, gx, gy, lam: float):
    """A29."""
    d = np.maximum(1.0, cell_pins(nl) + lam * nl.cell_w.astype(np.float64) * nl.cell_h.astype(np.float64))
    return gx / d, gy / d


def clamp(nl, x, y):
    """A33: lower-left corners kept inside the region."""
    return (np.clip(x, nl.xl, nl.xh - nl.cell_w.astype(np.float64)),
            np.clip(y, nl.yl, nl.yh - nl.cell_h.astype(np.float64)))


def nesterov_step(u, v, vp, g, gp, a, alpha_prev, clamp_fn):
    """A28 on flat vectors: returns (u_new, v_new, a_new, alpha)."""
    num = math.sqrt(float(np.sum((v - vp) ** 2)))
    den = math.sqrt(float(np.sum((g - gp) ** 2)))
    alpha = num / den if den > 0 else alpha_prev
    u_new = clamp_fn(v - alpha * g)
    a_new = (1.0 + math.sqrt(4.0 * a * a + 1.0)) / 2.0
    v_new = clamp_fn(u_new + (a - 1.0) / a_new * (u_new - u))
    return u_new, v_new, a_new, alpha


# -------------------------------------------------------------------------------- the loop
@dataclasses.dataclass
class GpState:
    u: np.ndarray      # [2, N] major solution
    v: np.ndarray      # [2, N] reference solution (gradient evaluated here)
    vp: np.ndarray     # v_{k-1}
    g: np.ndarray      # preconditioned gradient at v
    gp: np.ndarray     # ... at v_{k-1}
    a: float
    lam: float
    gamma: float
    hpwl: float
    tau: float
    alpha: float
    k: int
    frozen: bool = False


def _eval_pre(nl, x, y, gamma, lam):
    r = evaluate(nl, x, y, gamma, lam, with_hpwl=True)
    gx, gy = precondition(nl, r["gx"], r["gy"], lam)
    return np.stack([gx, gy]), r


def gp_init(nl, x0, y0, prm: GpParams | None = None) -> GpState:
    prm = prm or GpParams()
    x, y = clamp(nl, np.asarray(x0, np.float64), np.asarray(y0, np.float64))
    tau = overflow(nl, density_map(nl, x, y), prm.target_density)
    gamma = gamma_of(nl, tau, prm)
    r = evaluate(nl, x, y, gamma, 1.0, with_hpwl=True)
    lam = prm.lambda_scale * (np.abs(r["wl_gx"]).sum() + np.abs(r["wl_gy"]).sum()) / \
        (np.abs(r["d_gx"]).sum() + np.abs(r["d_gy"]).sum())
    v = np.stack([x, y])
    g, r = _eval_pre(nl, x, y, gamma, lam)
    rms = math.sqrt(float(np.sum(g * g)) / g.size)
    eta = prm.init_rms_bins * nl.bin_w / rms if rms > 0 else 0.0
    vp = v - eta * g
    gp, _ = _eval_pre(nl, vp[0], vp[1], gamma, lam)
    return GpState(u=v.copy(), v=v, vp=vp, g=g, gp=gp, a=1.0, lam=float(lam), gamma=gamma,
                   hpwl=r["hpwl"], tau=tau, alpha=0.0, k=0)


def gp_step(nl, st: GpState, prm: GpParams | None = None) -> dict:
    """One GP iteration: Nesterov update (A28), evaluation at v_{k+1}, preconditioning (A29),
    overflow (A30), lambda (eq 18, A32) and gamma (A31) updates.  Mutates st; returns stats."""
    prm = prm or GpParams()

    def cl(z):
        return np.stack(clamp(nl, z[0], z[1]))

    if st.frozen:   # A36: converged; the state stays as it is
        r = evaluate(nl, st.v[0], st.v[1], st.gamma, st.lam, with_hpwl=True)
        stats = dict(k=st.k, hpwl=r["hpwl"], overflow=st.tau, lam=st.lam, gamma=st.gamma, obj=r["obj"],
                     alpha=st.alpha, wl=r["wl"])
        st.k += 1
        return stats
    u_new, v_new, a_new, alpha = nesterov_step(st.u, st.v, st.vp, st.g, st.gp, st.a, st.alpha, cl)
    g_new, r = _eval_pre(nl, v_new[0], v_new[1], st.gamma, st.lam)
    tau = overflow(nl, r["rho"], prm.target_density)
    p = (r["hpwl"] - st.hpwl) / prm.dhpwl_ref
    lam = min(st.lam * mu(p, st.k, prm), 1e30)
    stats = dict(k=st.k, hpwl=r["hpwl"], overflow=tau, lam=lam, gamma=gamma_of(nl, tau, prm),
                 obj=r["obj"], alpha=alpha, wl=r["wl"])
    st.vp, st.gp = st.v, st.g
    st.u, st.v, st.g, st.a = u_new, v_new, g_new, a_new
    st.lam, st.gamma, st.hpwl, st.tau, st.alpha = lam, stats["gamma"], r["hpwl"], tau, alpha
    st.k += 1
    st.frozen = tau < prm.stop_overflow
    return stats
