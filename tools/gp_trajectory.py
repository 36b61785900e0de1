"""GP-loop trajectories on the device (SURVEY §8f NEXT-1 measurement: iterations/s and the
HPWL / overflow trajectory) from the paper's initial placement.

    python tools/gp_trajectory.py [config ...] [--iters N]     (needs a B200)
"""
import argparse
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_dac_lindlrkp19_b200 as dp  # noqa: E402
from synth import make_netlist, make_positions  # noqa: E402


def run(name, iters, every, dhpwl_ref=None):
    nl = make_netlist(name)
    x, y = make_positions(nl, "initial")
    dev = torch.device("cuda", 0)
    xt, yt = torch.as_tensor(x, device=dev), torch.as_tensor(y, device=dev)
    ctx = dp.dp_create(nl)
    kw = {} if dhpwl_ref is None else {"dhpwl_ref": dhpwl_ref}
    loop = dp.GpLoop(ctx, max_history=iters, **kw)
    loop.init(xt, yt)
    loop.run(5)
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    loop.run(iters - 5)
    b.record()
    torch.cuda.synchronize()
    ms = a.elapsed_time(b) / (iters - 5)
    hist = loop.history(iters)
    print(f"== {name}: {nl.num_cells} cells, {nl.num_nets} nets, {nl.num_pins} pins, "
          f"{nl.bins_x}x{nl.bins_y} bins; {iters} iterations; {1e3 / ms:.1f} iterations/s "
          f"({ms * 1e3:.1f} us/iteration, device time, CUDA-graph replay); dhpwl_ref = "
          f"{loop.params.dhpwl_ref:g}")
    print(f"{'k':>6} {'HPWL':>14} {'overflow':>9} {'lambda':>11} {'gamma':>10} {'alpha':>10}")
    for h in hist:
        if int(h["k"]) % every == 0 or int(h["k"]) == iters - 1:
            print(f"{int(h['k']):6d} {h['hpwl']:14.6e} {h['overflow']:9.4f} {h['lam']:11.4e} {h['gamma']:10.3f} "
                  f"{h['alpha']:10.4f}")
    below = [int(h["k"]) for h in hist if h["overflow"] < 0.1]
    print(f"first iteration with overflow < 0.1: {below[0] if below else 'not reached'}")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="*", default=["adaptec1", "bigblue4"])
    ap.add_argument("--iters", type=int, default=2000)
    ap.add_argument("--every", type=int, default=100)
    ap.add_argument("--dhpwl-ref", type=float, default=None, help="eq-18 reference (default 3.5e5, P:450)")
    args = ap.parse_args()
    for c in args.configs:
        run(c, args.iters, args.every, args.dhpwl_ref)


if __name__ == "__main__":
    main()
