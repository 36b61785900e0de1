"""GPU parity of the LSE wirelength model (reading A27) through the C
ABI (dp_set_wl_model(DP_WL_LSE)) against the fp64 oracle, same tolerances as WA."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_dac_lindlrkp19_b200 as dp
from synth import custom_netlist, make_netlist, make_positions
from parity_util import check_scalar, check_vector, to_np

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def _t(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.float32), device=DEV)


@pytest.mark.parametrize("gscale", [0.05, 0.5, 5.0, 50.0])
@pytest.mark.parametrize("weighted", [False, True])
def test_lse_grad_tiny(gscale, weighted):
    nl = make_netlist("tiny")
    if weighted:
        nl.net_weight = np.random.default_rng(1).uniform(0.5, 2.0, nl.num_nets).astype(np.float32)
    ctx = dp.dp_create(nl)
    ctx.set_wl_model("lse")
    x, y = make_positions(nl)
    gamma = gscale * nl.bin_w
    out = ctx.wl_grad(_t(x), _t(y), gamma)
    wl, gx, gy = oracle.lse(nl, x, y, np.float32(gamma))
    check_scalar("LSE", out["wl"].item(), wl)
    check_vector("dLSE/dx", to_np(out["gx"]), gx)
    check_vector("dLSE/dy", to_np(out["gy"]), gy)


def test_lse_high_fanout_and_degenerate():
    """Every lanes-per-net class, the warp-per-net and CTA-per-net paths (up to 10K pins),
    degree 0/1 nets and a 2-pin net on one cell."""
    rng = np.random.default_rng(21)
    nc = 20000
    degs = [0, 1, 1, 2, 2, 3, 5, 8, 9, 16, 17, 31, 32, 33, 64, 65, 100, 128, 129, 200, 256, 257, 1000, 10000]
    degs = degs + list(rng.integers(2, 8, 3000))
    ns = np.concatenate([[0], np.cumsum(degs)])
    npins = int(ns[-1])
    p2c = rng.integers(0, nc, npins)
    p2c[ns[5]:ns[5] + 2] = 7
    w = rng.integers(2, 41, nc).astype(np.float32)
    h = np.full(nc, 12.0, np.float32)
    W = 8192.0
    nl = custom_netlist(ns, p2c, rng.random(npins) * w[p2c], rng.random(npins) * h[p2c], w, h,
                        (0, 0, W, W), (256, 256))
    ctx = dp.dp_create(nl)
    ctx.set_wl_model("lse")
    x = (rng.random(nc) * (W - w)).astype(np.float32)
    y = (rng.random(nc) * (W - h)).astype(np.float32)
    for gamma in (2.0, 40.0):
        out = ctx.wl_grad(_t(x), _t(y), gamma)
        wl, gx, gy = oracle.lse(nl, x, y, gamma)
        check_scalar("LSE", out["wl"].item(), wl)
        check_vector("dLSE/dx", to_np(out["gx"]), gx)
        check_vector("dLSE/dy", to_np(out["gy"]), gy)


@pytest.mark.parametrize("dist", ["spread", "initial"])
def test_eval_lse_with_hpwl(dist):
    """dp_eval with LSE: obj = LSE + lambda D, gradient, and the HPWL pass (bit-exact)."""
    nl = make_netlist("tiny")
    ctx = dp.dp_create(nl)
    x, y = make_positions(nl, dist)
    gamma = nl.bin_w
    ref = oracle.evaluate(nl, x, y, gamma, 0.5, wl_model="lse")
    ctx.set_wl_model("lse")
    out = ctx.eval(_t(x), _t(y), gamma, 0.5, with_hpwl=True)
    check_scalar("LSE", out["wl"].item(), ref["wl"])
    check_scalar("obj", out["obj"].item(), ref["obj"])
    assert out["hpwl"].item() == ref["hpwl"]
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    check_vector("gy", to_np(out["gy"]), ref["gy"])
    # switching back re-captures the evaluation graph: WA again
    ctx.set_wl_model("wa")
    out = ctx.eval(_t(x), _t(y), gamma, 0.5)
    check_scalar("WA", out["wl"].item(), oracle.wa(nl, x, y, gamma)[0])


def test_invalid_model():
    nl = make_netlist("tiny")
    ctx = dp.dp_create(nl)
    with pytest.raises(dp.DPError):
        ctx.set_wl_model(7)


@pytest.mark.slow
def test_lse_full_size_adaptec1():
    nl = make_netlist("adaptec1")
    ctx = dp.dp_create(nl)
    ctx.set_wl_model("lse")
    x, y = make_positions(nl)
    gamma = nl.bin_w
    out = ctx.wl_grad(_t(x), _t(y), gamma)
    wl, gx, gy = oracle.lse(nl, x, y, gamma)
    check_scalar("LSE", out["wl"].item(), wl)
    check_vector("dLSE/dx", to_np(out["gx"]), gx)
    check_vector("dLSE/dy", to_np(out["gy"]), gy)
