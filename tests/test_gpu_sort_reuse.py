"""GPU: the density sort is reused between evaluations.

The scatter keeps the tile-ordered list of small cells from the last sort; a cell that has left
the tile it is listed in (a stray) is scattered and gathered through the global int64 map and
field with the same arithmetic.  Every bin's int64 sum is order independent, so an evaluation
over a stale list is bit-identical to one over a fresh sort: these tests compare a context that
reuses its list (positions moved since its sort) with a context that sorts on every evaluation
(DP_REUSE_SORT=0), bit for bit, and with the oracle.  Requires a B200."""
import os

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


def _ctx(nl, **env):
    """A context with the given environment switches, in deterministic mode (the WA gradient as
    exact int64 sums, NEXT-2): the fp32 WA atomics would otherwise differ from call to call."""
    old = {k: os.environ.get(k) for k in env}
    os.environ.update({k: str(v) for k, v in env.items()})
    try:
        ctx = dp.dp_create(nl)
        dp.dp_set_deterministic(ctx, 1)
        return ctx
    finally:
        for k, v in old.items():
            if v is None:
                del os.environ[k]
            else:
                os.environ[k] = v


def _eval(ctx, x, y, nl):
    out = ctx.eval(_t(x), _t(y), nl.bin_w, 1.0)
    torch.cuda.synchronize()
    return {k: (v.clone() if torch.is_tensor(v) else v) for k, v in out.items()}


def _same(a, b):
    for k in ("obj", "wl", "energy"):
        assert a[k].item() == b[k].item(), (k, a[k].item(), b[k].item())
    assert torch.equal(a["gx"], b["gx"]) and torch.equal(a["gy"], b["gy"])


def _moves(nl, x, y, kind, seed=7):
    rng = np.random.default_rng(seed)
    W, H = nl.xh - nl.xl, nl.yh - nl.yl
    if kind == "jitter":        # a GP-like step: every cell moves ~0.5 bin
        return (x + rng.normal(0, 0.5 * nl.bin_w, x.shape)).astype(np.float32), \
               (y + rng.normal(0, 0.5 * nl.bin_h, y.shape)).astype(np.float32)
    if kind == "drift":         # a few bins: many cells change tiles
        return (x + rng.normal(0, 4.0 * nl.bin_w, x.shape)).astype(np.float32), \
               (y + rng.normal(0, 4.0 * nl.bin_h, y.shape)).astype(np.float32)
    if kind == "reshuffle":     # every cell somewhere else: (almost) all strays
        return make_positions(nl, "spread", seed=seed)
    if kind == "collapse":      # spread -> the P:153 'initial' clump (every walker's tile empties)
        return make_positions(nl, "initial")
    if kind == "outside":       # a tenth of the cells leave the region (empty footprints)
        xo, yo = x.copy(), y.copy()
        sel = rng.random(x.shape) < 0.1
        xo[sel] = nl.xh + 0.25 * W
        yo[sel] = nl.yl - 0.25 * H
        return xo, yo
    raise ValueError(kind)


@pytest.mark.parametrize("name", ["tiny", "adaptec1"])
@pytest.mark.parametrize("kind", ["jitter", "drift", "reshuffle", "collapse", "outside"])
@pytest.mark.parametrize("cond,rc", [(0, 0), (1, 0), (0, 1)])
def test_stale_list_bit_identical(name, kind, cond, rc):
    """cond = 1: the sort kernels inside a graph IF node (DP_SORT_COND=1), else early returns;
    rc = 1: the gather recomputes the footprints instead of reading the scatter's records."""
    nl = make_netlist(name)
    x0, y0 = make_positions(nl)
    x1, y1 = _moves(nl, x0, y0, kind)
    reuse = _ctx(nl, DP_REUSE_SORT=1, DP_RESORT_PCT=100, DP_SORT_COND=cond, DP_GATHER_RC=rc)   # keeps the list of x0
    fresh = _ctx(nl, DP_REUSE_SORT=0)
    _eval(reuse, x0, y0, nl)
    st0 = dp.dp_debug_sort_stats(reuse)
    a = _eval(reuse, x1, y1, nl)
    st1 = dp.dp_debug_sort_stats(reuse)
    assert st1["sorts"] == st0["sorts"] == 1          # the second evaluation did not sort
    # strays: cells whose first bin left the listed tile by more than the walkers' margin (tiny's
    # 64^2 map is one tile; a 0.5-bin jitter stays inside the margin; cells outside are empty)
    if name != "tiny" and kind not in ("outside", "jitter"):
        assert st1["strays_last"] > 0
    b = _eval(fresh, x1, y1, nl)
    _same(a, b)
    da, db = reuse.density_grad(_t(x1), _t(y1)), fresh.density_grad(_t(x1), _t(y1))
    assert da["energy"].item() == db["energy"].item()
    assert torch.equal(da["gx"], db["gx"]) and torch.equal(da["gy"], db["gy"])
    assert torch.equal(reuse.density_map(_t(x1), _t(y1)), fresh.density_map(_t(x1), _t(y1)))
    # and back: the cells return to the listed tiles (or further strays), still identical
    c = _eval(reuse, x0, y0, nl)
    d = _eval(fresh, x0, y0, nl)
    _same(c, d)
    if name == "tiny":
        ref = oracle.evaluate(nl, x1, y1, nl.bin_w, 1.0)
        check_scalar("WA", a["wl"].item(), ref["wl"])
        check_scalar("D", a["energy"].item(), ref["energy"])
        check_vector("gx", to_np(a["gx"]), ref["gx"])
        check_vector("gy", to_np(a["gy"]), ref["gy"])


def test_resort_threshold():
    """The list is rebuilt on the evaluation after one with more strays than DP_RESORT_PCT."""
    nl = make_netlist("adaptec1")
    x0, y0 = make_positions(nl)
    ctx = _ctx(nl, DP_REUSE_SORT=1, DP_RESORT_PCT=5)
    _eval(ctx, x0, y0, nl)
    assert dp.dp_debug_sort_stats(ctx)["sorts"] == 1
    _eval(ctx, x0, y0, nl)                       # same positions: no strays, no sort
    st = dp.dp_debug_sort_stats(ctx)
    assert st["sorts"] == 1 and st["strays_last"] == 0
    xj, yj = _moves(nl, x0, y0, "jitter")        # ~0.5 bin: inside the walkers' margin, no sort
    _eval(ctx, xj, yj, nl)
    st = dp.dp_debug_sort_stats(ctx)
    assert st["sorts"] == 1 and st["strays_last"] < 0.05 * nl.num_cells
    x1, y1 = _moves(nl, x0, y0, "reshuffle")
    _eval(ctx, x1, y1, nl)                       # evaluated over the stale list
    st = dp.dp_debug_sort_stats(ctx)
    assert st["sorts"] == 1 and st["strays_last"] > 0.05 * nl.num_cells
    _eval(ctx, x1, y1, nl)                       # this one re-sorts: no strays after it
    st = dp.dp_debug_sort_stats(ctx)
    assert st["sorts"] == 2 and st["strays_last"] == 0


@pytest.mark.slow
def test_bigblue4_trajectory_bit_identical():
    """A random walk of 0.5-bin steps at bigblue4 size (the bench's trajectory): each step's
    evaluation over the reused list equals a fresh sort's, bit for bit; sampled cells against
    the oracle's force on the last step."""
    nl = make_netlist("bigblue4")
    x, y = make_positions(nl)
    reuse = _ctx(nl)                          # bigblue4: reuse by default
    fresh = _ctx(nl, DP_REUSE_SORT=0)
    rng = np.random.default_rng(11)
    for k in range(6):
        a = _eval(reuse, x, y, nl)
        b = _eval(fresh, x, y, nl)
        _same(a, b)
        x = (x + rng.normal(0, 0.5 * nl.bin_w, x.shape)).astype(np.float32)
        y = (y + rng.normal(0, 0.5 * nl.bin_h, y.shape)).astype(np.float32)
    st = dp.dp_debug_sort_stats(reuse)
    assert st["sorts"] < 6


def test_fixed_cells_and_regions_request_a_sort():
    """dp_set_fixed builds the fixed-charge map with its own list and un-fixing changes the
    listed set: each requests a sort, and the evaluations match a sort-every-time context."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    reuse = _ctx(nl, DP_REUSE_SORT=1, DP_RESORT_PCT=100)
    fresh = _ctx(nl, DP_REUSE_SORT=0)
    _same(_eval(reuse, x, y, nl), _eval(fresh, x, y, nl))
    fixed = np.zeros(nl.num_cells, dtype=np.uint8)
    fixed[::7] = 1
    for c in (reuse, fresh):
        dp.dp_set_fixed(c, fixed, _t(x), _t(y))
    x1, y1 = _moves(nl, x, y, "drift")
    x1[fixed == 1], y1[fixed == 1] = x[fixed == 1], y[fixed == 1]
    _same(_eval(reuse, x1, y1, nl), _eval(fresh, x1, y1, nl))
    for c in (reuse, fresh):
        dp.dp_set_fixed(c, None, None, None)
    _same(_eval(reuse, x1, y1, nl), _eval(fresh, x1, y1, nl))
    assert dp.dp_debug_sort_stats(reuse)["sorts"] >= 3


def test_reuse_default():
    """Reuse is the default at every size: three evaluations at the same adaptec1
    positions sort once; DP_REUSE_SORT=0 sorts every time."""
    nl = make_netlist("adaptec1")
    x, y = make_positions(nl)
    ctx = dp.dp_create(nl)
    old = os.environ.get("DP_REUSE_SORT")
    os.environ["DP_REUSE_SORT"] = "0"
    try:
        ctx0 = dp.dp_create(nl)
    finally:
        if old is None:
            del os.environ["DP_REUSE_SORT"]
        else:
            os.environ["DP_REUSE_SORT"] = old
    for _ in range(3):
        ctx.eval(_t(x), _t(y), nl.bin_w, 1.0)
        ctx0.eval(_t(x), _t(y), nl.bin_w, 1.0)
    assert dp.dp_debug_sort_stats(ctx)["sorts"] == 1
    assert dp.dp_debug_sort_stats(ctx0)["sorts"] == 3
