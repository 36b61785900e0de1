"""Fixed cells (dp_set_fixed, SURVEY §8f NEXT-4 "fixed macros"; reading A34): the precomputed
fixed-charge map plus the movable cells' map equals the map of all cells bit for bit (int64),
the evaluation matches the oracle with fixed cells' gradients 0, and the GP loop leaves fixed
cells where they are."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_dac_lindlrkp19_b200 as dp
from synth import make_netlist, make_positions
from parity_util import check_scalar, check_vector, to_np

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def _t(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.float32), device=DEV)


def _mask(nl, frac, seed):
    """Every large block plus a random fraction of the standard cells."""
    rng = np.random.default_rng(seed)
    big = (nl.cell_w > 2 * nl.bin_w) | (nl.cell_h > 2 * nl.bin_h)
    return big | (rng.random(nl.num_cells) < frac)


@pytest.mark.parametrize("name,frac", [("tiny", 0.1), ("tiny", 0.0), ("adaptec1", 0.02)])
@pytest.mark.parametrize("dist", ["spread", "initial"])
def test_fixed_map_is_exact(name, frac, dist):
    nl = make_netlist(name)
    x, y = make_positions(nl, dist)
    xt, yt = _t(x), _t(y)
    ctx = dp.dp_create(nl)
    full = ctx.density_map(xt, yt).clone()
    m = _mask(nl, frac, 5)
    dp.dp_set_fixed(ctx, m, xt, yt)
    part = ctx.density_map(xt, yt)
    torch.cuda.synchronize()
    assert torch.equal(full, part)


@pytest.mark.parametrize("dist", ["spread", "initial"])
@pytest.mark.parametrize("model", ["wa", "lse"])
def test_fixed_eval_parity(dist, model):
    nl = make_netlist("tiny")
    x, y = make_positions(nl, dist)
    xt, yt = _t(x), _t(y)
    m = _mask(nl, 0.15, 6)
    ctx = dp.dp_create(nl)
    ctx.set_wl_model(model)
    dp.dp_set_fixed(ctx, m, xt, yt)
    out = ctx.eval(xt, yt, nl.bin_w, 0.7, with_hpwl=True)
    ref = oracle.evaluate(nl, x, y, nl.bin_w, 0.7, wl_model=model, fixed=m)
    check_scalar("WL", out["wl"].item(), ref["wl"])
    check_scalar("D", out["energy"].item(), ref["energy"])
    check_scalar("obj", out["obj"].item(), ref["obj"])
    assert out["hpwl"].item() == ref["hpwl"]
    gx, gy = to_np(out["gx"]), to_np(out["gy"])
    assert np.all(gx[m] == 0.0) and np.all(gy[m] == 0.0)
    check_vector("gx", gx, ref["gx"])
    check_vector("gy", gy, ref["gy"])
    # deterministic mode honours the mask too
    dp.dp_set_deterministic(ctx, True)
    out2 = ctx.eval(xt, yt, nl.bin_w, 0.7)
    check_vector("gx det", to_np(out2["gx"]), ref["gx"])
    # clearing the mask restores the plain evaluation
    dp.dp_set_deterministic(ctx, False)
    dp.dp_set_fixed(ctx, None)
    out3 = ctx.eval(xt, yt, nl.bin_w, 0.7)
    ref3 = oracle.evaluate(nl, x, y, nl.bin_w, 0.7, wl_model=model)
    check_vector("gx cleared", to_np(out3["gx"]), ref3["gx"])


def test_fixed_full_size_parity():
    """bigblue4-shaped netlist with its large blocks fixed (as macros are): parity on a sample of
    cells and the scalars, in bench.py's configuration."""
    nl = make_netlist("bigblue4")
    x, y = make_positions(nl)
    xt, yt = _t(x), _t(y)
    m = _mask(nl, 0.0, 7)
    assert m.sum() > 100
    ctx = dp.dp_create(nl)
    dp.dp_set_fixed(ctx, m, xt, yt)
    out = ctx.eval(xt, yt, nl.bin_w, 1.0)
    ref = oracle.evaluate(nl, x, y, nl.bin_w, 1.0, with_hpwl=False, fixed=m)
    check_scalar("D", out["energy"].item(), ref["energy"])
    check_scalar("obj", out["obj"].item(), ref["obj"])
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    check_vector("gy", to_np(out["gy"]), ref["gy"])


def test_gp_keeps_fixed_cells():
    nl = make_netlist("tiny")
    x, y = make_positions(nl, "initial")
    m = _mask(nl, 0.05, 8)
    # fixed cells spread over the region (as placed macros would be)
    rng = np.random.default_rng(9)
    x = x.copy()
    y = y.copy()
    x[m] = rng.uniform(nl.xl, nl.xh - nl.cell_w[m]).astype(np.float32)
    y[m] = rng.uniform(nl.yl, nl.yh - nl.cell_h[m]).astype(np.float32)
    xt, yt = _t(x), _t(y)
    ctx = dp.dp_create(nl)
    dp.dp_set_fixed(ctx, m, xt, yt)
    loop = dp.GpLoop(ctx)
    loop.init(xt, yt)
    loop.run(300)
    hist = loop.history()
    ux, uy = loop.positions()
    ux, uy = ux.cpu().numpy(), uy.cpu().numpy()
    assert np.array_equal(ux[m], x[m]) and np.array_equal(uy[m], y[m])
    assert hist[-1]["overflow"] < hist[0]["overflow"]
    assert np.abs(ux[~m] - x[~m]).max() > nl.bin_w   # movable cells did move


def test_gp_overflow_with_fixed_macros():
    """A30 with fixed macros (A34): the loop's overflow at the start point equals the
    oracle's — fixed charge counted at the target density, normalised by the movable area."""
    from oracle import gp as ogp
    nl = make_netlist("adaptec1")
    x, y = make_positions(nl, "spread")
    m = _mask(nl, 0.0, 1)
    assert m.any()
    ctx = dp.dp_create(nl)
    dp.dp_set_fixed(ctx, m, _t(x), _t(y))
    loop = dp.GpLoop(ctx, target_density=0.9)
    loop.init(_t(x), _t(y))
    _, sc = loop.debug_state()
    rho = oracle.density_map(nl, x, y, 1)
    cells = np.nonzero(m)[0]
    from synth import custom_netlist
    fixed_nl = custom_netlist([0], [], [], [], nl.cell_w[cells], nl.cell_h[cells], (nl.xl, nl.yl, nl.xh, nl.yh),
                              (nl.bins_x, nl.bins_y))
    rho_f = oracle.density_map(fixed_nl, x[cells], y[cells], 1)
    ref = ogp.overflow(nl, rho, 0.9, m, rho_f)
    assert abs(sc["tau"] - ref) <= 1e-5 * max(ref, 1e-3), (sc["tau"], ref)


def test_gp_recaptures_after_set_fixed():
    """dp_set_* after the loop captured its iteration graph: the next dp_gp_run
    re-captures, so cells fixed after 5 iterations stay where they are from then on."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl, "initial")
    ctx = dp.dp_create(nl)
    loop = dp.GpLoop(ctx)
    loop.init(_t(x), _t(y))
    loop.run(5)
    ux, uy = loop.positions()
    m = _mask(nl, 0.05, 8)
    dp.dp_set_fixed(ctx, m, ux, uy)
    ux0, uy0 = ux.cpu().numpy().copy(), uy.cpu().numpy().copy()
    loop.run(20)
    ux1, uy1 = loop.positions()
    ux1, uy1 = ux1.cpu().numpy(), uy1.cpu().numpy()
    assert np.array_equal(ux1[m], ux0[m]) and np.array_equal(uy1[m], uy0[m])
    assert np.abs(ux1[~m] - ux0[~m]).max() > 0.0


def test_gp_with_fillers_and_fixed_macros():
    """ePlace-style setup (reading A35): pinless fillers bring the movable area to 90% of the
    free area, the large blocks are fixed; the device loop spreads movable cells and fillers.
    The evaluation with fillers matches the oracle (fillers are plain cells of the map)."""
    from synth import add_fillers
    nl0 = make_netlist("tiny")
    x0, y0 = make_positions(nl0, "initial")
    big = _mask(nl0, 0.0, 1)
    rng = np.random.default_rng(3)
    x0[big] = rng.uniform(nl0.xl, nl0.xh - nl0.cell_w[big]).astype(np.float32)
    y0[big] = rng.uniform(nl0.yl, nl0.yh - nl0.cell_h[big]).astype(np.float32)
    nl, x, y, fixed = add_fillers(nl0, x0, y0, 0.9, fixed=big)
    assert nl.num_cells > nl0.num_cells
    xt, yt = _t(x), _t(y)
    ctx = dp.dp_create(nl)
    dp.dp_set_fixed(ctx, fixed, xt, yt)
    out = ctx.eval(xt, yt, nl.bin_w, 0.3)
    ref = oracle.evaluate(nl, x, y, nl.bin_w, 0.3, with_hpwl=False, fixed=fixed)
    check_scalar("obj", out["obj"].item(), ref["obj"])
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    loop = dp.GpLoop(ctx, target_density=0.9)
    loop.init(xt, yt)
    loop.run(600)
    hist = loop.history()
    print([(int(h["k"]), round(h["overflow"], 3)) for h in hist[::100]])
    assert hist[-1]["overflow"] < 0.5 * hist[0]["overflow"]
