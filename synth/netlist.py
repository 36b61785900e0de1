"""Seeded synthetic netlists shaped like the paper's benchmarks.

This module is the ONE piece shared by the oracle side and the CUDA side (tests, bench).
It holds none of the method's arithmetic (no wirelength, density, transform or gradient
math): it only draws hypergraphs, cell sizes, placement regions and positions.

Recipe.  The paper prints no netlist
statistics, so every distribution below is a stated assumption calibrated to the cell /
net / pin counts of the configs in BASELINE.json:

* net degrees: truncated power law P(d) ~ d^-alpha on [2, d_max]; alpha solved by
  bisection so that the mean degree equals N_p / N_e; the sampled degrees are then nudged
  by +-1 (from the last net backwards, staying inside [2, d_max]) until sum(d) == N_p.
* pin -> cell: every net draws a centre cell c0 ~ U[0, N_c); each pin picks
  (c0 + round(N(0, 64^2))) mod N_c with probability 0.9, else a uniform cell.
* cells: standard cells of height 12 and integer width U{2..40}; a fraction 3e-4 (at
  least one once N_c >= 100k) are large blocks with sides ~ U[96, 1024].
* region: square, W = H = sqrt(sum(w h) / 0.6) rounded up to a multiple of the bin
  count M (utilisation ~0.6), lower-left corner at (0, 0).
* pin offsets: dx ~ U[0, w], dy ~ U[0, h] relative to the cell's lower-left corner.
* positions: "spread" - lower-left ~ U[0, W - w] x U[0, H - h]; "initial" - centres
  ~ N(W/2, (0.001 W)^2) per axis (the paper's random initial placement, PAPER.md
  Sec. III: cells at the layout centre with noise of 0.1% of the region size).

Seeds: netlist seed = 1000 + config index, position seed = 2000 + config index +
100 * distribution index (spread = 0, initial = 1).
"""
from __future__ import annotations

import dataclasses
import math

import numpy as np

__all__ = ["Netlist", "CONFIGS", "make_netlist", "make_positions", "config_by_name",
           "solve_alpha", "custom_netlist", "add_fillers"]


@dataclasses.dataclass
class Netlist:
    """CSR hypergraph + cell geometry + bin grid. All arrays are numpy, C-contiguous."""
    name: str
    num_cells: int
    num_nets: int
    num_pins: int
    net_start: np.ndarray     # int32 [num_nets + 1]
    pin2cell: np.ndarray      # int32 [num_pins]   (pins stored in net order)
    pin_dx: np.ndarray        # float32 [num_pins] offset from the cell's lower-left corner
    pin_dy: np.ndarray        # float32 [num_pins]
    cell_w: np.ndarray        # float32 [num_cells]
    cell_h: np.ndarray        # float32 [num_cells]
    xl: float
    yl: float
    xh: float
    yh: float
    bins_x: int
    bins_y: int
    net_weight: np.ndarray | None = None   # float32 [num_nets] or None (= 1)

    @property
    def bin_w(self) -> float:
        return (self.xh - self.xl) / self.bins_x

    @property
    def bin_h(self) -> float:
        return (self.yh - self.yl) / self.bins_y

    def degrees(self) -> np.ndarray:
        return np.diff(self.net_start)


# name, N_c, N_e, N_p, M, d_max
CONFIGS = [
    dict(name="tiny", cells=1_000, nets=1_200, pins=4_000, bins=64, d_max=64),
    dict(name="adaptec1", cells=211_000, nets=221_000, pins=944_000, bins=512, d_max=2500),
    dict(name="bigblue4", cells=2_180_000, nets=2_230_000, pins=8_900_000, bins=1024, d_max=4000),
    # industrial: N_e from design6's net/cell ratio, 4.0 pins/net assumed
    dict(name="industrial", cells=10_000_000, nets=10_230_000, pins=40_920_000, bins=2048, d_max=4000),
]


def config_by_name(name: str) -> tuple[int, dict]:
    for i, c in enumerate(CONFIGS):
        if c["name"] == name:
            return i, c
    raise KeyError(name)


def _powerlaw_pmf(alpha: float, d_max: int) -> tuple[np.ndarray, np.ndarray]:
    d = np.arange(2, d_max + 1, dtype=np.float64)
    w = d ** (-alpha)
    return d, w / w.sum()


def solve_alpha(mean: float, d_max: int) -> float:
    """Exponent of the truncated power law on [2, d_max] whose mean is `mean`."""
    lo, hi = 0.5, 12.0
    for _ in range(100):
        mid = 0.5 * (lo + hi)
        d, p = _powerlaw_pmf(mid, d_max)
        if (d * p).sum() > mean:
            lo = mid
        else:
            hi = mid
    return 0.5 * (lo + hi)


def _sample_degrees(rng: np.random.Generator, nets: int, pins: int, d_max: int) -> np.ndarray:
    alpha = solve_alpha(pins / nets, d_max)
    d, p = _powerlaw_pmf(alpha, d_max)
    cdf = np.cumsum(p)
    deg = (np.searchsorted(cdf, rng.random(nets), side="right") + 2).astype(np.int64)
    deg = np.minimum(deg, d_max)
    diff = pins - int(deg.sum())
    # nudge from the last net backwards, one pin per net per pass
    while diff != 0:
        step = 1 if diff > 0 else -1
        ok = (deg < d_max) if step > 0 else (deg > 2)
        idx = np.nonzero(ok)[0][::-1][: abs(diff)]
        if idx.size == 0:
            raise ValueError("cannot realise pin count with these degree bounds")
        deg[idx] += step
        diff -= step * idx.size
    return deg


def _cells(rng: np.random.Generator, cells: int) -> tuple[np.ndarray, np.ndarray]:
    w = rng.integers(2, 41, size=cells).astype(np.float32)
    h = np.full(cells, 12.0, dtype=np.float32)
    n_big = int(round(3e-4 * cells))
    if cells >= 100_000:
        n_big = max(1, n_big)
    if n_big:
        big = rng.choice(cells, size=n_big, replace=False)
        w[big] = rng.uniform(96, 1024, size=n_big).astype(np.float32)
        h[big] = rng.uniform(96, 1024, size=n_big).astype(np.float32)
    return w, h


def make_netlist(name_or_cfg, extra_fanout: tuple[int, ...] = (), bins: int | None = None,
                 seed: int | None = None) -> Netlist:
    """Build the synthetic netlist for a BASELINE config (by name or dict).

    `extra_fanout` appends nets of the given degrees (the high-fanout sweep), taking their
    pins from 2-pin nets so N_p stays fixed.  `bins` overrides the bin count (the
    bin-resolution sweep)."""
    if isinstance(name_or_cfg, str):
        idx, cfg = config_by_name(name_or_cfg)
    else:
        cfg = name_or_cfg
        idx = cfg.get("index", 99)
    rng = np.random.default_rng(1000 + idx if seed is None else seed)
    nc, ne, npins, d_max = cfg["cells"], cfg["nets"], cfg["pins"], cfg["d_max"]
    deg = _sample_degrees(rng, ne, npins, d_max)
    if extra_fanout:
        need = int(sum(extra_fanout))
        two = np.nonzero(deg == 2)[0]
        # removing k two-pin nets frees 2k pins; add the fanout nets, then rebalance
        k = need // 2
        keep = np.ones(ne, dtype=bool)
        keep[two[:k]] = False
        deg = np.concatenate([deg[keep], np.array(extra_fanout, dtype=np.int64)])
        diff = npins - int(deg.sum())
        j = deg.size - len(extra_fanout) - 1
        while diff != 0:
            if diff > 0:
                deg[j] += 1; diff -= 1
            elif deg[j] > 2:
                deg[j] -= 1; diff += 1
            j -= 1
        ne = deg.size
    net_start = np.zeros(ne + 1, dtype=np.int64)
    np.cumsum(deg, out=net_start[1:])
    assert net_start[-1] == npins
    # pin -> cell with locality around a per-net centre
    c0 = rng.integers(0, nc, size=ne)
    centre = np.repeat(c0, deg)
    near = np.rint(rng.normal(0.0, 64.0, size=npins)).astype(np.int64)
    uni = rng.integers(0, nc, size=npins)
    pick_uniform = rng.random(npins) < 0.1
    pin2cell = np.where(pick_uniform, uni, (centre + near) % nc).astype(np.int32)
    w, h = _cells(rng, nc)
    pin_dx = (rng.random(npins, dtype=np.float32) * w[pin2cell]).astype(np.float32)
    pin_dy = (rng.random(npins, dtype=np.float32) * h[pin2cell]).astype(np.float32)
    m = cfg["bins"] if bins is None else bins
    area = float(np.sum(w.astype(np.float64) * h.astype(np.float64)))
    side = math.sqrt(area / 0.6)
    side = float(math.ceil(side / m) * m)
    return Netlist(name=cfg["name"], num_cells=nc, num_nets=ne, num_pins=npins,
                   net_start=net_start.astype(np.int32), pin2cell=pin2cell,
                   pin_dx=pin_dx, pin_dy=pin_dy, cell_w=w, cell_h=h,
                   xl=0.0, yl=0.0, xh=side, yh=side, bins_x=m, bins_y=m)


def make_positions(nl: Netlist, distribution: str = "spread", config_index: int | None = None,
                   seed: int | None = None) -> tuple[np.ndarray, np.ndarray]:
    """Cell lower-left corners (float32) for the 'spread' or 'initial' distribution."""
    dist_idx = {"spread": 0, "initial": 1}[distribution]
    if config_index is None:
        try:
            config_index = config_by_name(nl.name)[0]
        except KeyError:
            config_index = 99
    rng = np.random.default_rng(2000 + config_index + 100 * dist_idx if seed is None else seed)
    W = nl.xh - nl.xl
    H = nl.yh - nl.yl
    w = nl.cell_w.astype(np.float64)
    h = nl.cell_h.astype(np.float64)
    if distribution == "spread":
        x = nl.xl + rng.random(nl.num_cells) * np.maximum(W - w, 0.0)
        y = nl.yl + rng.random(nl.num_cells) * np.maximum(H - h, 0.0)
    else:
        x = nl.xl + rng.normal(W / 2, 0.001 * W, size=nl.num_cells) - w / 2
        y = nl.yl + rng.normal(H / 2, 0.001 * H, size=nl.num_cells) - h / 2
    return x.astype(np.float32), y.astype(np.float32)


def custom_netlist(net_start, pin2cell, pin_dx, pin_dy, cell_w, cell_h, region, bins,
                   name="custom", net_weight=None) -> Netlist:
    """Wrap hand-built arrays (tests) into a Netlist with the right dtypes."""
    net_start = np.ascontiguousarray(net_start, dtype=np.int32)
    return Netlist(name=name, num_cells=int(len(cell_w)), num_nets=int(len(net_start) - 1),
                   num_pins=int(net_start[-1]),
                   net_start=net_start,
                   pin2cell=np.ascontiguousarray(pin2cell, dtype=np.int32),
                   pin_dx=np.ascontiguousarray(pin_dx, dtype=np.float32),
                   pin_dy=np.ascontiguousarray(pin_dy, dtype=np.float32),
                   cell_w=np.ascontiguousarray(cell_w, dtype=np.float32),
                   cell_h=np.ascontiguousarray(cell_h, dtype=np.float32),
                   xl=float(region[0]), yl=float(region[1]), xh=float(region[2]), yh=float(region[3]),
                   bins_x=int(bins[0]), bins_y=int(bins[1]),
                   net_weight=None if net_weight is None else np.ascontiguousarray(net_weight, dtype=np.float32))


def add_fillers(nl: Netlist, x: np.ndarray, y: np.ndarray, target_density: float = 1.0,
                fixed: np.ndarray | None = None, seed: int = 4242):
    """Append pinless filler cells (ePlace's whitespace fillers; reading A35) so that
    movable + filler area = target_density * (region area - fixed area).  Filler size: the mean
    width of the movable standard cells (sides <= 2 bins) x their row height 12.  Fillers start
    where the movable cells are (uniform over the movable cells' bounding box).  Returns
    (netlist, x, y, fixed) with the fillers appended after the original cells (no pins)."""
    rng = np.random.default_rng(seed)
    fx = np.zeros(nl.num_cells, dtype=bool) if fixed is None else np.asarray(fixed, dtype=bool)
    area = nl.cell_w.astype(np.float64) * nl.cell_h.astype(np.float64)
    region = (nl.xh - nl.xl) * (nl.yh - nl.yl)
    free = target_density * (region - area[fx].sum()) - area[~fx].sum()
    std = (~fx) & (nl.cell_w <= 2 * nl.bin_w) & (nl.cell_h <= 2 * nl.bin_h)
    fw = float(np.mean(nl.cell_w[std])) if std.any() else nl.bin_w
    fh = 12.0
    n = max(0, int(free // (fw * fh)))
    mv = ~fx
    lo_x, hi_x = float(x[mv].min()), float((x[mv] + nl.cell_w[mv]).max())
    lo_y, hi_y = float(y[mv].min()), float((y[mv] + nl.cell_h[mv]).max())
    xf = (lo_x + rng.random(n) * max(hi_x - lo_x - fw, 0.0)).astype(np.float32)
    yf = (lo_y + rng.random(n) * max(hi_y - lo_y - fh, 0.0)).astype(np.float32)
    out = dataclasses.replace(
        nl, name=nl.name + "+fillers", num_cells=nl.num_cells + n,
        cell_w=np.concatenate([nl.cell_w, np.full(n, fw, np.float32)]),
        cell_h=np.concatenate([nl.cell_h, np.full(n, fh, np.float32)]))
    return (out, np.concatenate([x, xf]).astype(np.float32), np.concatenate([y, yf]).astype(np.float32),
            np.concatenate([fx, np.zeros(n, dtype=bool)]))
