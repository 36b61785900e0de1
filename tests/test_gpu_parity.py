"""GPU parity: the CUDA path through the C ABI against the fp64 oracle on the same seeded
inputs (BASELINE.json north_star tolerances; HPWL bit-exact).  Requires a B200."""
import numpy as np
import pytest
import torch

import oracle
import paper_conf_dac_lindlrkp19_b200 as dp
from synth import custom_netlist, make_netlist, make_positions
from parity_util import check_map, check_scalar, check_vector, to_np

pytestmark = pytest.mark.gpu
DEV = torch.device("cuda", 0)


def _t(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.float32), device=DEV)


@pytest.fixture(scope="module")
def tiny():
    nl = make_netlist("tiny")
    return nl, dp.dp_create(nl)


# ------------------------------------------------------------------------------ transforms
@pytest.mark.parametrize("m", [16, 64, 256])
def test_transforms(m):
    nl = custom_netlist([0], [], [], [], [1.0], [1.0], (0, 0, 10.0 * m, 7.0 * m), (m, m))
    ctx = dp.dp_create(nl)
    rng = np.random.default_rng(m)
    a = rng.standard_normal((m, m))
    inp = _t(a)
    a32 = to_np(inp)
    got = to_np(ctx.transform(dp.DP_T_DCT2, inp))
    check_map("DCT2", got, oracle.dct2(a32))
    got = to_np(ctx.transform(dp.DP_T_IDCT2, inp))
    check_map("IDCT2", got, oracle.transform(oracle.IDCT, oracle.transform(oracle.IDCT, a32, 1), 0))
    got = to_np(ctx.transform(dp.DP_T_IDXST_IDCT, inp))
    check_map("IDXST_IDCT", got, oracle.transform(oracle.IDXST, oracle.transform(oracle.IDCT, a32, 1), 0))
    got = to_np(ctx.transform(dp.DP_T_IDCT_IDXST, inp))
    check_map("IDCT_IDXST", got, oracle.transform(oracle.IDCT, oracle.transform(oracle.IDXST, a32, 1), 0))


def test_transforms_rectangular():
    nl = custom_netlist([0], [], [], [], [1.0], [1.0], (0, 0, 320.0, 90.0), (32, 128))
    ctx = dp.dp_create(nl)
    a = np.random.default_rng(3).standard_normal((32, 128))
    inp = _t(a)
    a32 = to_np(inp)
    check_map("DCT2", to_np(ctx.transform(dp.DP_T_DCT2, inp)), oracle.dct2(a32))
    check_map("IDXST_IDCT", to_np(ctx.transform(dp.DP_T_IDXST_IDCT, inp)),
              oracle.transform(oracle.IDXST, oracle.transform(oracle.IDCT, a32, 1), 0))


# ---------------------------------------------------------------------------- density map
@pytest.mark.parametrize("dist", ["spread", "initial"])
def test_density_map_tiny(tiny, dist):
    nl, ctx = tiny
    x, y = make_positions(nl, dist)
    got = to_np(ctx.density_map(_t(x), _t(y)))
    # tile bins resolve 2^-29 (two 32-bit words per bin): the map is fp32-accurate
    check_map("rho", got, oracle.density_map(nl, x, y, 1), rel=2e-6)


def test_fields_tiny(tiny):
    nl, ctx = tiny
    x, y = make_positions(nl)
    rho = oracle.density_map(nl, x, y, 1)
    f = ctx.fields(_t(rho))
    rho32 = rho.astype(np.float32).astype(np.float64)
    psi, xi_x, xi_y = oracle.fields(nl, oracle.dct2(rho32))
    check_map("psi", to_np(f["psi"]), psi)
    check_map("xi_x", to_np(f["xi_x"]), xi_x)
    check_map("xi_y", to_np(f["xi_y"]), xi_y)
    check_scalar("energy", f["energy"].item(), oracle.energy(nl, rho32, psi))


@pytest.mark.parametrize("mx,my", [(16, 16), (32, 32), (64, 64), (128, 128), (256, 256), (512, 512), (1024, 1024),
                                   (32, 128), (256, 64), (64, 1024), (2048, 2048)])
def test_fields_sizes(mx, my):
    """The three CTA-FFT passes (P1 rows, P2 columns + energy, P3 rows; fields.cu) on random maps
    of every radix plan of the radix-16 core (16, 32 = 16 x 2, 64 = 16 x 4, 128 = 16 x 8,
    256 = 16^2, 512 = 16^2 x 2, 1024 = 16^2 x 4, 2048 = 16^2 x 8), square and rectangular, against
    eqs 9a-9d via the naive eq 7a/7b/8a."""
    W, H = 10.0 * mx, 7.0 * my
    nl = custom_netlist([0], [], [], [], [1.0], [1.0], (0, 0, W, H), (mx, my))
    ctx = dp.dp_create(nl)
    rho = np.random.default_rng(mx * 7 + my).random((mx, my)) * 2.0
    f = ctx.fields(_t(rho))
    rho32 = rho.astype(np.float32).astype(np.float64)
    psi, xi_x, xi_y = oracle.fields(nl, oracle.dct2(rho32))
    check_map("xi_x", to_np(f["xi_x"]), xi_x)
    check_map("xi_y", to_np(f["xi_y"]), xi_y)
    check_scalar("energy", f["energy"].item(), oracle.energy(nl, rho32, psi))


# ------------------------------------------------------------------------------ wirelength
@pytest.mark.parametrize("gscale", [0.05, 0.5, 5.0, 50.0])
@pytest.mark.parametrize("weighted", [False, True])
def test_wl_grad_tiny(gscale, weighted):
    nl = make_netlist("tiny")
    if weighted:
        nl.net_weight = np.random.default_rng(1).uniform(0.5, 2.0, nl.num_nets).astype(np.float32)
    ctx = dp.dp_create(nl)
    x, y = make_positions(nl)
    gamma = gscale * nl.bin_w
    out = ctx.wl_grad(_t(x), _t(y), gamma)
    wl, gx, gy = oracle.wa(nl, x, y, np.float32(gamma))
    check_scalar("WA", out["wl"].item(), wl)
    check_vector("dWA/dx", to_np(out["gx"]), gx)
    check_vector("dWA/dy", to_np(out["gy"]), gy)


def test_wl_grad_high_fanout_and_degenerate():
    """Every lanes-per-net class, a 10K-pin net (CTA-per-net path), degree 0/1 nets, repeated
    cells inside a net, nets spanning the whole region."""
    rng = np.random.default_rng(11)
    nc = 20000
    degs = [0, 1, 1, 2, 2, 3, 5, 8, 9, 16, 17, 31, 32, 33, 64, 65, 100, 128, 129, 200, 256, 257, 1000, 10000]
    degs = degs + list(rng.integers(2, 8, 3000))
    ns = np.concatenate([[0], np.cumsum(degs)])
    npins = int(ns[-1])
    p2c = rng.integers(0, nc, npins)
    p2c[ns[5]:ns[5] + 2] = 7  # a 2-pin net on one cell (coincident pins)
    w = rng.integers(2, 41, nc).astype(np.float32)
    h = np.full(nc, 12.0, np.float32)
    W = 8192.0
    nl = custom_netlist(ns, p2c, rng.random(npins) * w[p2c], rng.random(npins) * h[p2c], w, h,
                        (0, 0, W, W), (256, 256))
    ctx = dp.dp_create(nl)
    x = (rng.random(nc) * (W - w)).astype(np.float32)
    y = (rng.random(nc) * (W - h)).astype(np.float32)
    for gamma in (2.0, 40.0):
        out = ctx.wl_grad(_t(x), _t(y), gamma)
        wl, gx, gy = oracle.wa(nl, x, y, gamma)
        check_scalar("WA", out["wl"].item(), wl)
        check_vector("dWA/dx", to_np(out["gx"]), gx)
        check_vector("dWA/dy", to_np(out["gy"]), gy)
    assert ctx.hpwl(_t(x), _t(y)).item() == oracle.hpwl(nl, x, y)


def test_empty_and_degree_one_netlists():
    nl = custom_netlist([0, 1, 1], [3], [0.5], [0.5], np.full(10, 4.0), np.full(10, 4.0), (0, 0, 160, 160), (16, 16))
    ctx = dp.dp_create(nl)
    x = np.linspace(0, 150, 10).astype(np.float32)
    y = np.linspace(5, 120, 10).astype(np.float32)
    out = ctx.eval(_t(x), _t(y), 2.0, 0.5, with_hpwl=True)
    assert out["wl"].item() == 0.0 and out["hpwl"].item() == 0.0
    ref = oracle.evaluate(nl, x, y, 2.0, 0.5)
    check_scalar("energy", out["energy"].item(), ref["energy"])
    check_vector("gx", to_np(out["gx"]), ref["gx"])


# -------------------------------------------------------------------------------- HPWL
@pytest.mark.parametrize("name", ["tiny", "adaptec1", "bigblue4"])
@pytest.mark.parametrize("dist", ["spread", "initial"])
def test_hpwl_bit_exact(name, dist):
    nl = make_netlist(name)
    ctx = dp.dp_create(nl)
    x, y = make_positions(nl, dist)
    got = ctx.hpwl(_t(x), _t(y)).item()
    assert got == oracle.hpwl(nl, x, y)   # bit-exact fp64 (reading A7)
    out = ctx.eval(_t(x), _t(y), nl.bin_w, 1.0, with_hpwl=True)
    assert out["hpwl"].item() == got


def test_hpwl_extreme_magnitudes():
    """Coordinates spanning 2^-20 .. 2^40 exercise every limb of the fixed-point sum."""
    rng = np.random.default_rng(5)
    nc = 4000
    ns = np.arange(0, 2 * 1500 + 1, 2)
    p2c = rng.integers(0, nc, ns[-1])
    dx = (rng.random(ns[-1]) * 2.0 ** rng.integers(-20, 4, ns[-1])).astype(np.float32)
    nl = custom_netlist(ns, p2c, dx, dx[::-1].copy(), np.ones(nc), np.ones(nc), (0, 0, 1e13, 1e13), (16, 16))
    ctx = dp.dp_create(nl)
    x = (2.0 ** rng.uniform(-20, 40, nc)).astype(np.float32)
    y = (2.0 ** rng.uniform(-20, 40, nc)).astype(np.float32)
    assert ctx.hpwl(_t(x), _t(y)).item() == oracle.hpwl(nl, x, y)


# ------------------------------------------------------------------------- density grad
@pytest.mark.parametrize("dist", ["spread", "initial"])
def test_density_grad_tiny(tiny, dist):
    nl, ctx = tiny
    x, y = make_positions(nl, dist)
    out = ctx.density_grad(_t(x), _t(y))
    D, gx, gy, _ = oracle.density(nl, x, y, 1)
    check_scalar("D", out["energy"].item(), D)
    check_vector("dD/dx", to_np(out["gx"]), gx)
    check_vector("dD/dy", to_np(out["gy"]), gy)


def _macro_netlist(stretch_bins=64):
    rng = np.random.default_rng(21)
    nc = 6000
    w = rng.integers(2, 41, nc).astype(np.float32)
    h = np.full(nc, 12.0, np.float32)
    big = rng.choice(nc, 12, replace=False)
    w[big] = rng.uniform(96, 700, 12).astype(np.float32)
    h[big] = rng.uniform(96, 700, 12).astype(np.float32)
    w[:5] = 0.0  # zero-area cells
    deg = rng.integers(2, 6, 7000)
    ns = np.concatenate([[0], np.cumsum(deg)])
    p2c = rng.integers(0, nc, ns[-1])
    W = 3200.0
    nl = custom_netlist(ns, p2c, rng.random(ns[-1]) * w[p2c], rng.random(ns[-1]) * h[p2c], w, h, (0, 0, W, W),
                        (stretch_bins, stretch_bins))
    x = (rng.random(nc) * (W - w)).astype(np.float32)
    y = (rng.random(nc) * (W - h)).astype(np.float32)
    x[5:40] = rng.uniform(-300, W + 200, 35)  # partly / fully outside the region (reading A11)
    return nl, x, y


@pytest.mark.parametrize("stretch", [0, 1])
def test_density_grad_macros_and_edges(stretch):
    nl, x, y = _macro_netlist()
    ctx = dp.dp_create(nl, stretch=stretch)
    out = ctx.density_grad(_t(x), _t(y))
    D, gx, gy, parts = oracle.density(nl, x, y, stretch)
    check_map("rho", to_np(ctx.density_map(_t(x), _t(y))), parts["rho"], rel=2e-6)
    check_scalar("D", out["energy"].item(), D)
    check_vector("dD/dx", to_np(out["gx"]), gx)
    check_vector("dD/dy", to_np(out["gy"]), gy)


# ------------------------------------------------------------------------------ full eval
@pytest.mark.parametrize("dist", ["spread", "initial"])
@pytest.mark.parametrize("lam", [0.0, 1e-4, 1.0])
def test_eval_tiny(dist, lam):
    nl = make_netlist("tiny")
    ctx = dp.dp_create(nl)
    x, y = make_positions(nl, dist)
    gamma = nl.bin_w
    out = ctx.eval(_t(x), _t(y), gamma, lam, with_hpwl=True)
    ref = oracle.evaluate(nl, x, y, gamma, lam)
    check_scalar("WA", out["wl"].item(), ref["wl"])
    check_scalar("D", out["energy"].item(), ref["energy"])
    check_scalar("obj", out["obj"].item(), ref["obj"])
    assert out["hpwl"].item() == ref["hpwl"]
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    check_vector("gy", to_np(out["gy"]), ref["gy"])


def test_eval_repeatable_and_stream_independent(tiny):
    """g2 is reset by every evaluation: repeated calls give the same result within fp32
    atomic-order noise; a side stream works the same as the default stream."""
    nl, ctx = tiny
    x, y = make_positions(nl)
    xt, yt = _t(x), _t(y)
    a = ctx.eval(xt, yt, 11.0, 0.3)
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        b = ctx.eval(xt, yt, 11.0, 0.3, stream=s)
    # no host sync between: the context orders its own calls across streams
    c = ctx.eval(xt, yt, 11.0, 0.3)
    torch.cuda.synchronize()
    ref = oracle.evaluate(nl, x, y, 11.0, 0.3)
    for o in (a, b, c):
        check_vector("gx", to_np(o["gx"]), ref["gx"])
        check_scalar("obj", o["obj"].item(), ref["obj"])
    check_vector("repeat gx", to_np(b["gx"]), to_np(a["gx"]), rel_l2=1e-5, rel_entry=1e-4)


def test_eval_host_e2e(tiny):
    nl, ctx = tiny
    x, y = make_positions(nl)
    gx = np.zeros(nl.num_cells, np.float32)
    gy = np.zeros(nl.num_cells, np.float32)
    sc = np.zeros(4)
    dp.dp_eval_host(ctx, x, y, 9.0, 0.5, gx, gy, sc, with_hpwl=True)
    torch.cuda.synchronize()
    ref = oracle.evaluate(nl, x, y, 9.0, 0.5)
    check_scalar("obj", sc[0], ref["obj"])
    assert sc[3] == ref["hpwl"]
    check_vector("gx", gx, ref["gx"])


@pytest.mark.parametrize("name", ["tiny", "adaptec1"])
def test_eval_host_async_pipeline(name):
    """dp_eval_host_async: six calls in flight on alternating staging slots, each with its own
    positions and pinned result buffers, equal bit for bit (deterministic mode) to synchronous
    dp_eval_host calls; the tiny case also against the oracle."""
    nl = make_netlist(name)
    ctx = dp.dp_create(nl)
    dp.dp_set_deterministic(ctx, 1)
    rng = np.random.default_rng(5)
    x0, y0 = make_positions(nl)
    pos = [((x0 + rng.normal(0, 2 * nl.bin_w, x0.shape)).astype(np.float32),
            (y0 + rng.normal(0, 2 * nl.bin_h, y0.shape)).astype(np.float32)) for _ in range(6)]
    hx = [torch.as_tensor(p[0]).pin_memory() for p in pos]
    hy = [torch.as_tensor(p[1]).pin_memory() for p in pos]
    out = [(torch.zeros(nl.num_cells).pin_memory(), torch.zeros(nl.num_cells).pin_memory(),
            torch.zeros(4, dtype=torch.float64).pin_memory()) for _ in pos]
    for k in range(len(pos)):
        dp.dp_eval_host_async(ctx, hx[k], hy[k], nl.bin_w, 0.5, out[k][0], out[k][1], out[k][2], True)
    dp.dp_eval_host_wait(ctx)
    for k in range(len(pos)):
        gx = np.zeros(nl.num_cells, np.float32)
        gy = np.zeros(nl.num_cells, np.float32)
        sc = np.zeros(4)
        dp.dp_eval_host(ctx, pos[k][0], pos[k][1], nl.bin_w, 0.5, gx, gy, sc, with_hpwl=True)
        assert np.array_equal(out[k][0].numpy(), gx) and np.array_equal(out[k][1].numpy(), gy), k
        assert out[k][2].numpy().tolist() == sc.tolist(), k
    if name == "tiny":
        ref = oracle.evaluate(nl, pos[3][0], pos[3][1], nl.bin_w, 0.5)
        check_scalar("obj", out[3][2][0].item(), ref["obj"])
        assert out[3][2][3].item() == ref["hpwl"]
        check_vector("gx", out[3][0].numpy(), ref["gx"])
        check_vector("gy", out[3][1].numpy(), ref["gy"])


@pytest.mark.slow
@pytest.mark.parametrize("name", ["adaptec1", "bigblue4"])
def test_eval_full_size(name):
    """BASELINE configs at full size in the launch configuration bench.py times."""
    nl = make_netlist(name)
    ctx = dp.dp_create(nl)
    x, y = make_positions(nl)
    gamma = nl.bin_w
    out = ctx.eval(_t(x), _t(y), gamma, 1.0, with_hpwl=True)
    ref = oracle.evaluate(nl, x, y, gamma, 1.0)
    check_scalar("WA", out["wl"].item(), ref["wl"])
    check_scalar("D", out["energy"].item(), ref["energy"])
    assert out["hpwl"].item() == ref["hpwl"]
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    check_vector("gy", to_np(out["gy"]), ref["gy"])


@pytest.mark.parametrize("env", [{"DP_WA_SPLIT": "50"}, {"DP_FFT": "2"}, {"DP_FFT": "1"}, {"DP_FUSE_COMBINE": "1"},
                                 {"DP_FUSE_COMBINE": "1", "DP_REUSE_SORT": "1"}, {"DP_GATHER_RC": "1"},
                                 {"DP_GATHER_RC": "1", "DP_REUSE_SORT": "1", "DP_FUSE_COMBINE": "1"}])
def test_schedule_switches_match(env):
    """The measured-and-off A/B switches of the evaluation schedule compute the
    same evaluation: the WA launch split around the transforms (the same work units and partial
    slots in two launches), the hybrid and the CTA-FFT field paths at 512^2 — against the default
    context (WA / D / HPWL / gradient) and the oracle."""
    import os
    nl = make_netlist("adaptec1")
    x, y = make_positions(nl)
    xt, yt = _t(x), _t(y)
    base = dp.dp_create(nl)
    a = base.eval(xt, yt, nl.bin_w, 1.0, with_hpwl=True)
    a = {k: (v.clone() if torch.is_tensor(v) else v) for k, v in a.items()}
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    try:
        ctx = dp.dp_create(nl)
    finally:
        for k, v in old.items():
            if v is None:
                del os.environ[k]
            else:
                os.environ[k] = v
    b = ctx.eval(xt, yt, nl.bin_w, 1.0, with_hpwl=True)
    torch.cuda.synchronize()
    assert b["hpwl"].item() == a["hpwl"].item()
    if "DP_WA_SPLIT" in env:   # same field path: D bit-identical; WA partial slots identical
        assert b["energy"].item() == a["energy"].item()
        assert b["wl"].item() == a["wl"].item()
    check_scalar("WA", b["wl"].item(), a["wl"].item())
    check_scalar("D", b["energy"].item(), a["energy"].item())
    check_vector("gx", to_np(b["gx"]), to_np(a["gx"]))
    check_vector("gy", to_np(b["gy"]), to_np(a["gy"]))
    ref = oracle.evaluate(nl, x, y, nl.bin_w, 1.0)
    check_scalar("D (oracle)", b["energy"].item(), ref["energy"])
    check_vector("gx (oracle)", to_np(b["gx"]), ref["gx"])


@pytest.mark.slow
@pytest.mark.parametrize("name", ["adaptec1", "bigblue4"])
def test_initial_full_size(name):
    """The 'initial' placement (centres ~ N(W/2, (0.001 W)^2), every cell in a few bins)
    at full size: the density map (every walker in one tile, the wrap carry of the scatter's
    32-bit accumulators), the force gather where opposite fields cancel, and the full
    evaluation, against the oracle."""
    nl = make_netlist(name)
    ctx = dp.dp_create(nl)
    x, y = make_positions(nl, "initial")
    xt, yt = _t(x), _t(y)
    ref = oracle.evaluate(nl, x, y, nl.bin_w, 1.0)
    check_map("rho", to_np(ctx.density_map(xt, yt)), ref["rho"], rel=2e-6)
    d = ctx.density_grad(xt, yt)
    check_scalar("D", d["energy"].item(), ref["energy"])
    check_vector("dD/dx", to_np(d["gx"]), ref["d_gx"])
    check_vector("dD/dy", to_np(d["gy"]), ref["d_gy"])
    out = ctx.eval(xt, yt, nl.bin_w, 1.0, with_hpwl=True)
    check_scalar("WA", out["wl"].item(), ref["wl"])
    check_scalar("obj", out["obj"].item(), ref["obj"])
    assert out["hpwl"].item() == ref["hpwl"]
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    check_vector("gy", to_np(out["gy"]), ref["gy"])


@pytest.mark.slow
@pytest.mark.parametrize("gscale,lam", [(0.05, 1.0), (50.0, 1.0), (1.0, 0.0)])
def test_adaptec1_gamma_lambda_sweep(gscale, lam):
    """SURVEY §8(d) parity sweep at adaptec1 full size (211K cells: every WA path — window and
    far cells, warp-per-net and CTA-per-net big nets — not just the tiny config's one window):
    gamma in {0.05, 50} b and lambda = 0."""
    nl = make_netlist("adaptec1")
    ctx = dp.dp_create(nl)
    x, y = make_positions(nl)
    gamma = gscale * nl.bin_w
    out = ctx.eval(_t(x), _t(y), gamma, lam, with_hpwl=True)
    ref = oracle.evaluate(nl, x, y, gamma, lam)
    check_scalar("WA", out["wl"].item(), ref["wl"])
    check_scalar("obj", out["obj"].item(), ref["obj"])
    assert out["hpwl"].item() == ref["hpwl"]
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    check_vector("gy", to_np(out["gy"]), ref["gy"])


def test_invalid_args(tiny):
    nl, ctx = tiny
    x, y = make_positions(nl)
    gx = torch.empty(nl.num_cells, device=DEV)
    with pytest.raises(dp.DPError, match="INVALID_ARG"):
        dp.dp_eval(ctx, _t(x), _t(y), 0.0, 1.0, gx, gx.clone())
    with pytest.raises(dp.DPError, match="INVALID_ARG"):
        dp.dp_eval(ctx, _t(x), _t(y), 1.0, -1.0, gx, gx.clone())
    with pytest.raises(dp.DPError, match="INVALID_ARG"):
        dp.dp_eval(ctx, None, _t(y), 1.0, 1.0, gx, gx.clone())


@pytest.mark.parametrize("dist", ["spread", "initial"])
def test_density_bitwise_deterministic(tiny, dist):
    """The bin map accumulates in int64 fixed point, so the density energy and
    gradient are bitwise identical from call to call regardless of atomic order."""
    nl, ctx = tiny
    x, y = make_positions(nl, dist)
    a = ctx.density_grad(_t(x), _t(y))
    b = ctx.density_grad(_t(x), _t(y))
    assert a["energy"].item() == b["energy"].item()
    assert torch.equal(a["gx"], b["gx"]) and torch.equal(a["gy"], b["gy"])
    assert torch.equal(ctx.density_map(_t(x), _t(y)), ctx.density_map(_t(x), _t(y)))


@pytest.mark.parametrize("world", [2, 3])
def test_virtual_shards_reassemble(world):
    """dp_create_dist with no NCCL id (collectives skipped) on one GPU, one context per rank: the
    net / cell partition must reassemble the single-context results — WA and its
    gradient (each rank's partial gradient over all cells: the sum the reduce-scatter forms),
    HPWL, and the int64 bin map of each rank's cell block summing to the full map."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    gamma = nl.bin_w
    full = dp.dp_create(nl)
    ref = full.wl_grad(_t(x), _t(y), gamma)
    ref_map = full.density_map(_t(x), _t(y)).double()
    wl = 0.0
    hp = 0.0
    gx = torch.zeros(nl.num_cells, dtype=torch.float64, device=DEV)
    gy = torch.zeros_like(gx)
    rho = torch.zeros_like(ref_map)
    covered = np.zeros(nl.num_cells, np.int64)
    for r in range(world):
        cb, ce, _ = dp.dp_partition_plan(nl, r, world)
        covered[cb:ce] += 1
        ctx = dp.dp_create_dist(nl, 0, r, world, None)
        out = ctx.wl_grad(_t(x), _t(y), gamma)
        wl += out["wl"].item()
        gx += out["gx"].double()
        gy += out["gy"].double()
        hp += ctx.hpwl(_t(x), _t(y)).item()
        rho += ctx.density_map(_t(x), _t(y)).double()
    assert (covered == 1).all()
    check_scalar("WA", wl, ref["wl"].item(), rel=1e-6)
    # the gradient sums (fp32 atomics, different per-rank flush order): the oracle's bar
    check_vector("dWA/dx", to_np(gx), to_np(ref["gx"]))
    check_vector("dWA/dy", to_np(gy), to_np(ref["gy"]))
    assert hp == pytest.approx(oracle.hpwl(nl, x, y), rel=1e-14)
    check_map("rho", to_np(rho), to_np(ref_map), rel=1e-6)


@pytest.mark.parametrize("name", ["tiny", "adaptec1"])
def test_one_rank_nccl_context(name):
    """dp_create_dist with world = 1 and a real NCCL id: the distributed path with every collective
    (bin-map all-reduce, WA partial and HPWL-limb all-reduces, NCCL loaded with dlopen) runs on
    one GPU; it must equal the single context: bit-identical density map, HPWL and energy (exact
    or fixed-order), oracle parity for the rest."""
    nl = make_netlist(name)
    x, y = make_positions(nl)
    xt, yt = _t(x), _t(y)
    single = dp.dp_create(nl)
    a = single.eval(xt, yt, nl.bin_w, 1.0, with_hpwl=True)
    a = {k: (v.clone() if torch.is_tensor(v) else v) for k, v in a.items()}
    ctx = dp.dp_create_dist(nl, 0, 0, 1, dp.dp_nccl_unique_id())
    b = ctx.eval(xt, yt, nl.bin_w, 1.0, with_hpwl=True)
    torch.cuda.synchronize()
    assert b["hpwl"].item() == a["hpwl"].item() == oracle.hpwl(nl, x, y)
    assert b["energy"].item() == a["energy"].item()
    assert torch.equal(ctx.density_map(xt, yt), single.density_map(xt, yt))
    check_scalar("WA", b["wl"].item(), a["wl"].item(), rel=1e-6)
    check_vector("gx", to_np(b["gx"]), to_np(a["gx"]))
    check_vector("gy", to_np(b["gy"]), to_np(a["gy"]))


@pytest.mark.slow
@pytest.mark.parametrize("bins", [256, 2048, 4096])
def test_bin_sweep_density(bins):
    """BASELINE configs[4] (bin-resolution sweep): the bigblue4 netlist on 256^2..4096^2 maps —
    the shared-memory transform path above 1024 — density energy and gradient vs the oracle."""
    nl = make_netlist("bigblue4", bins=bins)
    x, y = make_positions(nl)
    ctx = dp.dp_create(nl)
    out = ctx.density_grad(_t(x), _t(y))
    D, fx, fy, _ = oracle.density(nl, x, y, 1)
    check_scalar("D", out["energy"].item(), D)
    check_vector("dD/dx", to_np(out["gx"]), fx)
    check_vector("dD/dy", to_np(out["gy"]), fy)


@pytest.mark.slow
def test_high_fanout_sweep():
    """BASELINE configs[4] (high-fanout sweep): bigblue4 with extra nets of 1K, 2K, 5K and 10K
    pins — WA, its gradient and HPWL vs the oracle."""
    nl = make_netlist("bigblue4", extra_fanout=(1000, 2000, 5000, 10000))
    x, y = make_positions(nl)
    ctx = dp.dp_create(nl)
    gamma = nl.bin_w
    out = ctx.wl_grad(_t(x), _t(y), gamma)
    wl, gx, gy = oracle.wa(nl, x, y, gamma)
    check_scalar("WA", out["wl"].item(), wl)
    check_vector("dWA/dx", to_np(out["gx"]), gx)
    check_vector("dWA/dy", to_np(out["gy"]), gy)
    assert ctx.hpwl(_t(x), _t(y)).item() == oracle.hpwl(nl, x, y)


@pytest.mark.slow
def test_eval_industrial():
    """BASELINE configs[3] shape on one GPU (10M cells, 10.23M nets, 40.9M pins, 2048^2 bins): the
    full evaluation vs the oracle."""
    nl = make_netlist("industrial")
    x, y = make_positions(nl)
    ctx = dp.dp_create(nl)
    gamma = nl.bin_w
    out = ctx.eval(_t(x), _t(y), gamma, 1.0, with_hpwl=True)
    ref = oracle.evaluate(nl, x, y, gamma, 1.0)
    check_scalar("WA", out["wl"].item(), ref["wl"])
    check_scalar("D", out["energy"].item(), ref["energy"])
    assert out["hpwl"].item() == ref["hpwl"]
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    check_vector("gy", to_np(out["gy"]), ref["gy"])


@pytest.mark.parametrize("bins,world", [(256, 2), (256, 4), (2048, 2), (2048, 8)])
def test_sharded_poisson_emulated_bit_identical(bins, world):
    """The row-sharded Poisson solve (P1 on each rank's rows, all-to-all, P2 on its
    columns, all-to-all, P3 on its rows) with `world` ranks emulated on one GPU: the same
    kernels on per-rank layouts must reproduce the unsharded solve bit for bit (every 1-D
    transform sees the same inputs in the same order; the energy slots are per column slab),
    and the oracle."""
    nl = custom_netlist([0], [], [], [], [1.0], [1.0], (0, 0, 10.0 * bins, 10.0 * bins), (bins, bins))
    import os
    os.environ["DP_FFT"] = "1"   # the CTA-FFT passes also at 256
    try:
        ctx = dp.dp_create(nl)
    finally:
        del os.environ["DP_FFT"]
    rho = np.random.default_rng(bins + world).random((bins, bins)) * 2.0
    ref = ctx.fields(_t(rho), want_psi=False)
    ref = {k: (v.clone() if torch.is_tensor(v) else v) for k, v in ref.items()}
    sh = dp.dp_debug_sharded_fields(ctx, world, _t(rho))
    assert torch.equal(sh["xi_x"], ref["xi_x"]) and torch.equal(sh["xi_y"], ref["xi_y"])
    assert sh["energy"].item() == ref["energy"].item()
    if bins <= 256:
        rho32 = rho.astype(np.float32).astype(np.float64)
        psi, xi_x, xi_y = oracle.fields(nl, oracle.dct2(rho32))
        check_map("xi_x", to_np(sh["xi_x"]), xi_x)
        check_scalar("energy", sh["energy"].item(), oracle.energy(nl, rho32, psi))


def test_one_rank_nccl_sharded_poisson():
    """A one-rank NCCL context on a 2048^2 map takes the row-sharded solve (reduce-scatter of the
    map, two all-to-alls, all-gather of the field through NCCL, here with one rank): the
    evaluation equals the single context bit for bit in energy and HPWL, and the gradient."""
    nl = make_netlist("adaptec1", bins=2048)
    x, y = make_positions(nl)
    xt, yt = _t(x), _t(y)
    single = dp.dp_create(nl)
    a = single.eval(xt, yt, nl.bin_w, 1.0, with_hpwl=True)
    a = {k: (v.clone() if torch.is_tensor(v) else v) for k, v in a.items()}
    ctx = dp.dp_create_dist(nl, 0, 0, 1, dp.dp_nccl_unique_id())
    b = ctx.eval(xt, yt, nl.bin_w, 1.0, with_hpwl=True)
    torch.cuda.synchronize()
    assert b["energy"].item() == a["energy"].item()
    assert b["hpwl"].item() == a["hpwl"].item()
    check_vector("gx", to_np(b["gx"]), to_np(a["gx"]))
    check_vector("gy", to_np(b["gy"]), to_np(a["gy"]))
