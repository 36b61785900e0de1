import sys, os
sys.path.insert(0, "tests"); sys.path.insert(0, ".")
import numpy as np, torch
from test_gpu_sort_reuse import _ctx, _eval, _moves, _t
import paper_conf_dac_lindlrkp19_b200 as dp
from synth import make_netlist, make_positions
nl = make_netlist("adaptec1")
x0, y0 = make_positions(nl)
x1, y1 = _moves(nl, x0, y0, "jitter")
for cond in ("1", "0"):
    os.environ["DP_SORT_COND"] = cond
    reuse = _ctx(nl, DP_RESORT_PCT=100); fresh = _ctx(nl, DP_REUSE_SORT=0)
    _eval(reuse, x0, y0, nl); a = _eval(reuse, x1, y1, nl); b = _eval(fresh, x1, y1, nl)
    print("cond", cond, dp.dp_debug_sort_stats(reuse))
    for k in ("obj", "wl", "energy"): print(k, a[k].item(), b[k].item(), a[k].item() == b[k].item())
    for k in ("gx", "gy"):
        d = (a[k] - b[k]).abs(); print(k, "ndiff", int((d > 0).sum()), "max", float(d.max()))
    ma = reuse.density_map(_t(x1), _t(y1)); mb = fresh.density_map(_t(x1), _t(y1))
    d = (ma - mb).abs(); print("map ndiff", int((d > 0).sum()), float(d.max()))
    da, db = reuse.density_grad(_t(x1), _t(y1)), fresh.density_grad(_t(x1), _t(y1))
    for k in ("gx", "gy"):
        d = (da[k] - db[k]).abs(); idx = torch.nonzero(d > 0).flatten()[:5]
        print("dgrad", k, "ndiff", int((d > 0).sum()), float(d.max()), idx.tolist(), da[k][idx].tolist(), db[k][idx].tolist())
