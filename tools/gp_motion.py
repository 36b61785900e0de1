"""How far cells move per GP iteration, and what the density sort reuse does along a real GP
trajectory (the bench's trajectory step size comes from here).

For each config: the GP loop (dp_gp_*, from the paper's initial placement P:153) is run one
iteration at a time; per iteration the rms and median cell displacement in bins and the share of
small cells whose 64-bin density tile changed are recorded.  Then the whole trajectory is timed
with the sort reused (default) and re-sorted every evaluation (DP_REUSE_SORT=0), with the number
of sorts the reusing context performed.

    python tools/gp_motion.py [config ...] [--iters N]      (needs a B200)
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_dac_lindlrkp19_b200 as dp  # noqa: E402
from synth import make_netlist, make_positions  # noqa: E402


def ctx_with(nl, **env):
    old = {k: os.environ.get(k) for k in env}
    os.environ.update({k: str(v) for k, v in env.items()})
    try:
        return dp.dp_create(nl)
    finally:
        for k, v in old.items():
            if v is None:
                del os.environ[k]
            else:
                os.environ[k] = v


def motion(name, iters):
    nl = make_netlist(name)
    dev = torch.device("cuda", 0)
    x, y = make_positions(nl, "initial")
    xt, yt = torch.as_tensor(x, device=dev), torch.as_tensor(y, device=dev)
    ctx = dp.dp_create(nl)
    loop = dp.GpLoop(ctx, max_history=iters + 8)
    loop.init(xt, yt)
    px, py = loop.positions()
    tile_w, tile_h = 64 * nl.bin_w, 64 * nl.bin_h
    rows = []
    for k in range(iters):
        loop.run(1)
        qx, qy = loop.positions()
        dx = (qx - px) / nl.bin_w
        dy = (qy - py) / nl.bin_h
        d = torch.sqrt(dx * dx + dy * dy)
        changed = ((torch.floor((qx - nl.xl) / tile_w) != torch.floor((px - nl.xl) / tile_w)) |
                   (torch.floor((qy - nl.yl) / tile_h) != torch.floor((py - nl.yl) / tile_h)))
        rows.append((k, float(torch.sqrt((d * d).mean())), float(d.median()), float(changed.float().mean())))
        px, py = qx, qy
    hist = loop.history(iters + 8)
    st = dp.dp_debug_sort_stats(ctx)
    loop.close()
    return nl, rows, hist, st


def timed_run(nl, iters, **env):
    dev = torch.device("cuda", 0)
    x, y = make_positions(nl, "initial")
    ctx = ctx_with(nl, **env)
    loop = dp.GpLoop(ctx, max_history=iters + 8)
    loop.init(torch.as_tensor(x, device=dev), torch.as_tensor(y, device=dev))
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    loop.run(iters)
    b.record()
    torch.cuda.synchronize()
    st = dp.dp_debug_sort_stats(ctx)
    hist = loop.history(iters + 8)
    loop.close()
    return a.elapsed_time(b) / iters, st, hist[-1]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("configs", nargs="*", default=["adaptec1", "bigblue4"])
    ap.add_argument("--iters", type=int, default=1500)
    ap.add_argument("--every", type=int, default=100)
    ap.add_argument("--json", default=None)
    args = ap.parse_args()
    out = {}
    for name in args.configs:
        nl, rows, hist, st = motion(name, args.iters)
        print(f"== {name}: {args.iters} GP iterations from the initial placement (P:153)")
        print(f"{'k':>6} {'rms move (bins)':>16} {'median move':>12} {'tile changes':>13} {'overflow':>9}")
        for (k, rms, med, ch), h in zip(rows, hist):
            if k % args.every == 0 or k == args.iters - 1:
                print(f"{k:6d} {rms:16.4f} {med:12.4f} {ch:13.5f} {h['overflow']:9.4f}")
        rms_all = np.array([r[1] for r in rows])
        med_all = np.array([r[2] for r in rows])
        ch_all = np.array([r[3] for r in rows])
        print(f"median over iterations: rms move {np.median(rms_all):.4f} bins, median move "
              f"{np.median(med_all):.4f} bins, tile changes {np.median(ch_all):.5f} per iteration; "
              f"sorts {st['sorts']} in {args.iters} evaluations (one-at-a-time run)")
        ms_r, st_r, last_r = timed_run(nl, args.iters)
        ms_s, st_s, last_s = timed_run(nl, args.iters, DP_REUSE_SORT=0)
        print(f"whole trajectory, device time: sort reused {1e3 / ms_r:.1f} it/s ({ms_r * 1e3:.1f} us/it, "
              f"{st_r['sorts']} sorts) vs sorted every evaluation {1e3 / ms_s:.1f} it/s ({ms_s * 1e3:.1f} us/it); "
              f"final HPWL {last_r['hpwl']:.6e} / {last_s['hpwl']:.6e}, overflow {last_r['overflow']:.4f} / "
              f"{last_s['overflow']:.4f}")
        out[name] = {"iters": args.iters, "median_rms_move_bins": float(np.median(rms_all)),
                     "median_median_move_bins": float(np.median(med_all)),
                     "median_tile_change_frac": float(np.median(ch_all)),
                     "rms_move_by_iter": rms_all[::10].tolist(), "tile_change_by_iter": ch_all[::10].tolist(),
                     "reuse_it_per_s": 1e3 / ms_r, "reuse_sorts": st_r["sorts"],
                     "sort_every_it_per_s": 1e3 / ms_s}
    if args.json:
        with open(args.json, "w") as f:
            json.dump(out, f)


if __name__ == "__main__":
    main()
