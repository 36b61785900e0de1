"""Fence regions on the GPU (dp_set_regions, "multiple electric
fields, e.g., one for each region"; reading A38) against oracle.evaluate_regions."""
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


def _fences(nl, k, seed):
    """k disjoint fences on a k x 1 strip layout of the region (bin-unaligned edges), and a
    region per cell: cells whose centre lies in fence r belong to it, plus 5% moved at random."""
    rng = np.random.default_rng(seed)
    W, H = nl.xh - nl.xl, nl.yh - nl.yl
    boxes = []
    for r in range(k):
        x0 = nl.xl + W * (r + 0.13) / k
        boxes.append((x0, nl.yl + 0.21 * H, x0 + 0.61 * W / k, nl.yl + 0.77 * H))
    return boxes, rng


@pytest.mark.parametrize("name,k,dist", [("tiny", 2, "spread"), ("tiny", 1, "initial"), ("adaptec1", 3, "spread")])
def test_regions_match_oracle(name, k, dist):
    nl = make_netlist(name)
    x, y = make_positions(nl, dist)
    boxes, rng = _fences(nl, k, 5)
    cx, cy = x + 0.5 * nl.cell_w, y + 0.5 * nl.cell_h
    reg = np.zeros(nl.num_cells, np.int32)
    for r, b in enumerate(boxes):
        reg[(cx >= b[0]) & (cx < b[2]) & (cy >= b[1]) & (cy < b[3])] = r + 1
    moved = rng.random(nl.num_cells) < 0.05
    reg[moved] = rng.integers(0, k + 1, int(moved.sum()))
    ctx = dp.dp_create(nl)
    dp.dp_set_regions(ctx, boxes, reg)
    out = ctx.eval(_t(x), _t(y), nl.bin_w, 0.7)
    ref = oracle.evaluate_regions(nl, x, y, nl.bin_w, 0.7, boxes, reg)
    check_scalar("D", out["energy"].item(), ref["energy"])
    check_scalar("obj", out["obj"].item(), ref["obj"])
    check_vector("gx", to_np(out["gx"]), ref["gx"])
    check_vector("gy", to_np(out["gy"]), ref["gy"])
    # clearing the regions restores the plain evaluation
    dp.dp_set_regions(ctx, [], None)
    plain = ctx.eval(_t(x), _t(y), nl.bin_w, 0.7)
    check_scalar("D plain", plain["energy"].item(), oracle.evaluate(nl, x, y, nl.bin_w, 0.7, with_hpwl=False)["energy"])


def test_regions_in_gp_loop():
    """The GP loop over a context with fences (the evaluation graph re-captured per A38's
    passes) runs and lowers the objective's density part from the P:153 start."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl, "initial")
    boxes, _ = _fences(nl, 2, 7)
    reg = (np.arange(nl.num_cells) % 3).astype(np.int32)
    ctx = dp.dp_create(nl)
    dp.dp_set_regions(ctx, boxes, reg)
    loop = dp.GpLoop(ctx)
    loop.init(_t(x), _t(y))
    loop.run(60)
    h = loop.history()
    assert all(np.isfinite(r["obj"]) for r in h)
    assert h[-1]["overflow"] < h[0]["overflow"]
