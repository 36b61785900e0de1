"""Pins of the fence-region oracle (oracle.evaluate_regions, reading A38: one electric field per
region), CPU only."""
import numpy as np
import pytest

import oracle
from synth import make_netlist, make_positions


def test_blockage_area_and_shape():
    """Blockage of fence r = the area outside its box; of the default region = the fences' area;
    a box on bin edges gives 0/1 bins, a box on bin centres half bins."""
    nl = make_netlist("tiny")
    b = nl.bin_w
    boxes = [(nl.xl + 4 * b, nl.yl + 8 * b, nl.xl + 20 * b, nl.yl + 16 * b),
             (nl.xl + 30.5 * b, nl.yl + 2.5 * b, nl.xl + 40.5 * b, nl.yl + 12.5 * b)]
    abin = nl.bin_w * nl.bin_h
    W, H = nl.xh - nl.xl, nl.yh - nl.yl
    area = [(bx[2] - bx[0]) * (bx[3] - bx[1]) for bx in boxes]
    assert oracle.region_blockage(nl, boxes, 0).sum() * abin == pytest.approx(sum(area), rel=1e-12)
    for r in (1, 2):
        assert oracle.region_blockage(nl, boxes, r).sum() * abin == pytest.approx(W * H - area[r - 1], rel=1e-12)
    blk1 = oracle.region_blockage(nl, boxes, 1)
    assert set(np.unique(blk1)) == {0.0, 1.0}
    blk2 = oracle.region_blockage(nl, boxes, 2)
    assert blk2[30, 2] == pytest.approx(0.75) and blk2[30, 5] == pytest.approx(0.5) and blk2[33, 5] == 0.0


def test_whole_layout_fence_equals_plain_evaluation():
    """One fence covering the layout with every cell in it: the fence's blockage is 0, the
    default region is a uniform unit map (zero energy and field once the DC term is removed,
    A15), so the result is the plain evaluation."""
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    box = [(nl.xl, nl.yl, nl.xh, nl.yh)]
    ref = oracle.evaluate(nl, x, y, nl.bin_w, 0.3, with_hpwl=False)
    got = oracle.evaluate_regions(nl, x, y, nl.bin_w, 0.3, box, np.ones(nl.num_cells, int))
    assert got["energy"] == pytest.approx(ref["energy"], rel=1e-10)
    np.testing.assert_allclose(got["gx"], ref["gx"], rtol=1e-9, atol=1e-12 * np.abs(ref["gx"]).max())
    no_fence = oracle.evaluate_regions(nl, x, y, nl.bin_w, 0.3, [], np.zeros(nl.num_cells, int))
    assert no_fence["energy"] == pytest.approx(ref["energy"], rel=1e-12)


def test_fence_pushes_cells_inward_and_mirror_symmetry():
    """A cell of a fence sitting on the fence's left edge is pushed right (into the fence) by the
    blockage outside; mirroring the layout (x -> W - x - w, fence mirrored) flips the sign of
    the x gradient and keeps D."""
    nl = make_netlist("tiny")
    b = nl.bin_w
    box = (nl.xl + 16 * b, nl.yl + 16 * b, nl.xl + 48 * b, nl.yl + 48 * b)
    x, y = make_positions(nl)
    reg = np.zeros(nl.num_cells, int)
    reg[0] = 1
    x = x.astype(np.float64)
    y = y.astype(np.float64)
    x[0] = box[0] - 0.5 * nl.cell_w[0]
    y[0] = 0.5 * (box[1] + box[3])
    r = oracle.evaluate_regions(nl, x, y, b, 1.0, [box], reg)
    assert r["d_gx"][0] < 0            # descent direction -grad points into the fence
    W = nl.xh + nl.xl
    xm = W - x - nl.cell_w
    boxm = (W - box[2], box[1], W - box[0], box[3])
    m = oracle.evaluate_regions(nl, xm, y, b, 1.0, [boxm], reg)
    assert m["energy"] == pytest.approx(r["energy"], rel=1e-9)
    np.testing.assert_allclose(m["d_gx"], -r["d_gx"], rtol=1e-7, atol=1e-9 * np.abs(r["d_gx"]).max())
    np.testing.assert_allclose(m["d_gy"], r["d_gy"], rtol=1e-7, atol=1e-9 * np.abs(r["d_gy"]).max())
