"""Deterministic mode (dp_set_deterministic; the paper's future work P:706):
parity with the oracle is unchanged, and the gradient (hence a whole GP trajectory) is
bit-identical from run to run and across streams."""
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


@pytest.mark.parametrize("dist", ["spread", "initial"])
@pytest.mark.parametrize("model", ["wa", "lse"])
def test_det_parity_tiny(dist, model):
    nl = make_netlist("tiny")
    ctx = dp.dp_create(nl)
    dp.dp_set_deterministic(ctx, True)
    ctx.set_wl_model(model)
    x, y = make_positions(nl, dist)
    out = ctx.eval(_t(x), _t(y), nl.bin_w, 0.5, with_hpwl=True)
    ref = oracle.evaluate(nl, x, y, nl.bin_w, 0.5, wl_model=model)
    check_scalar("WL", out["wl"].item(), ref["wl"])
    check_scalar("obj", out["obj"].item(), ref["obj"])
    assert out["hpwl"].item() == ref["hpwl"]
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    check_vector("gy", to_np(out["gy"]), ref["gy"])


def test_det_high_fanout_parity():
    """Big nets (warp- and CTA-per-net paths) go through the per-pin int64 conversion."""
    nl = make_netlist("tiny", extra_fanout=(150, 1030))
    ctx = dp.dp_create(nl)
    dp.dp_set_deterministic(ctx, True)
    x, y = make_positions(nl)
    out = ctx.wl_grad(_t(x), _t(y), 2 * nl.bin_w)
    wl, gx, gy = oracle.wa(nl, x, y, np.float32(2 * nl.bin_w))
    check_scalar("WA", out["wl"].item(), wl)
    check_vector("gx", to_np(out["gx"]), gx)
    check_vector("gy", to_np(out["gy"]), gy)


@pytest.mark.parametrize("name", ["adaptec1", "bigblue4"])
def test_det_bitwise_repeatable(name):
    """Three evaluations (two streams) give bit-identical gradients and scalars; the
    non-deterministic path agrees with them within the parity tolerance."""
    nl = make_netlist(name)
    ctx = dp.dp_create(nl)
    x, y = make_positions(nl)
    xt, yt = _t(x), _t(y)
    fast = ctx.eval(xt, yt, nl.bin_w, 1.0)
    dp.dp_set_deterministic(ctx, True)
    outs = []
    side = torch.cuda.Stream()
    for k in range(3):
        st = side if k == 1 else None
        with torch.cuda.stream(st or torch.cuda.current_stream()):
            o = ctx.eval(xt, yt, nl.bin_w, 1.0, stream=st)
        torch.cuda.synchronize()
        outs.append({k2: v.clone() for k2, v in o.items() if torch.is_tensor(v)})
    for o in outs[1:]:
        assert torch.equal(o["gx"], outs[0]["gx"]) and torch.equal(o["gy"], outs[0]["gy"])
        assert torch.equal(o["scalars"][:3], outs[0]["scalars"][:3])
    check_vector("gx det vs fast", to_np(outs[0]["gx"]), to_np(fast["gx"]))
    check_scalar("obj det vs fast", outs[0]["obj"].item(), fast["obj"].item())
    n_diff = int((fast["gx"] != outs[0]["gx"]).sum())
    print(f"{name}: entries where the fp32-atomic path differs from the deterministic one: {n_diff}")


def test_det_gp_trajectory_bitwise():
    """The whole GP loop is deterministic in this mode: two runs from the same start give
    bit-identical histories and positions."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl, "initial")
    runs = []
    for _ in range(2):
        ctx = dp.dp_create(nl)
        dp.dp_set_deterministic(ctx, True)
        loop = dp.GpLoop(ctx)
        loop.init(_t(x), _t(y))
        loop.run(50)
        h = loop.history()
        ux, uy = loop.positions()
        runs.append((h, ux.cpu().numpy(), uy.cpu().numpy()))
        loop.close()
    (h0, x0, y0), (h1, x1, y1) = runs
    assert h0 == h1
    assert np.array_equal(x0, x1) and np.array_equal(y0, y1)


@pytest.mark.parametrize("world", [2, 3, 8])
def test_det_gradient_bitwise_across_world_sizes(world):
    """NEXT-2 across partitions: in deterministic mode the WA work units and their
    fixed-point scales do not depend on the number of ranks, so the exact int64
    partial gradients of `world` virtual shards sum (what the int64 reduce-scatter does) to the
    single context's accumulator bit for bit (the int64 bin map is exact for any partition:
    test_gpu_parity.py::test_virtual_shards_reassemble / test_one_rank_nccl_context)."""
    nl = make_netlist("adaptec1")
    x, y = make_positions(nl, "spread")
    xt, yt = _t(x), _t(y)
    single = dp.dp_create(nl)
    dp.dp_set_deterministic(single, True)
    single.wl_grad(xt, yt, nl.bin_w)
    ref = dp.dp_debug_wa_accumulator(single)[: nl.num_cells]
    acc = None
    for r in range(world):
        ctx = dp.dp_create_dist(nl, 0, r, world, None)
        dp.dp_set_deterministic(ctx, True)
        ctx.wl_grad(xt, yt, nl.bin_w)
        part = dp.dp_debug_wa_accumulator(ctx)[: nl.num_cells]
        acc = part.clone() if acc is None else acc + part
        ctx.close()
    assert torch.equal(acc, ref)
