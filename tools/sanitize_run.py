"""Workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): every entry
point of the C ABI once on the tiny config (and adaptec1 unless --tiny), including the GP loop,
fixed cells, LSE, deterministic mode and the CTA-FFT / sharded field passes."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_dac_lindlrkp19_b200 as dp  # noqa: E402
from synth import custom_netlist, make_netlist, make_positions  # noqa: E402

dev = torch.device("cuda", 0)


def t(a):
    return torch.as_tensor(np.ascontiguousarray(a, dtype=np.float32), device=dev)


names = ["tiny"] if "--tiny" in sys.argv else ["tiny", "adaptec1"]
for name in names:
    nl = make_netlist(name)
    for dist in ("spread", "initial"):
        x, y = make_positions(nl, dist)
        ctx = dp.dp_create(nl)
        ctx.eval(t(x), t(y), nl.bin_w, 1.0, with_hpwl=True)
        ctx.wl_grad(t(x), t(y), nl.bin_w)
        ctx.density_grad(t(x), t(y))
        ctx.hpwl(t(x), t(y))
        ctx.set_wl_model("lse")
        ctx.eval(t(x), t(y), nl.bin_w, 1.0, with_hpwl=True)
        ctx.set_wl_model("wa")
        dp.dp_set_deterministic(ctx, True)
        ctx.eval(t(x), t(y), nl.bin_w, 1.0)
        dp.dp_set_deterministic(ctx, False)
        big = (nl.cell_w > 2 * nl.bin_w) | (nl.cell_h > 2 * nl.bin_h)
        dp.dp_set_fixed(ctx, big | (np.arange(nl.num_cells) % 17 == 0), t(x), t(y))
        ctx.eval(t(x), t(y), nl.bin_w, 1.0)
        dp.dp_set_fixed(ctx, None)
        if name == "tiny":
            loop = dp.GpLoop(ctx)
            loop.init(t(x), t(y))
            loop.run(3)
            loop.history()
            loop.close()
        torch.cuda.synchronize()
        ctx.close()
    # virtual shards (net-partitioned WA) and the emulated row-sharded solve on a small map
    x, y = make_positions(nl)
    for r in range(2):
        sh = dp.dp_create_dist(nl, 0, r, 2, None)
        sh.eval(t(x), t(y), nl.bin_w, 1.0, with_hpwl=True)
        torch.cuda.synchronize()
        sh.close()
import os  # noqa: E402
# the kept density list (round 2, second session): strays after moves, cells leaving the region, the IF-node
# variant, and the pipelined host path
for name in names:
    nl = make_netlist(name)
    x, y = make_positions(nl)
    rng = np.random.default_rng(1)
    for cond in ("0", "1"):
        os.environ["DP_REUSE_SORT"] = "1"
        os.environ["DP_RESORT_PCT"] = "100"
        os.environ["DP_SORT_COND"] = cond
        ctx = dp.dp_create(nl)
        for k in ("DP_REUSE_SORT", "DP_RESORT_PCT", "DP_SORT_COND"):
            del os.environ[k]
        ctx.eval(t(x), t(y), nl.bin_w, 1.0)
        x1 = (x + rng.normal(0, 4 * nl.bin_w, x.shape)).astype(np.float32)
        y1 = (y + rng.normal(0, 4 * nl.bin_h, y.shape)).astype(np.float32)
        ctx.eval(t(x1), t(y1), nl.bin_w, 1.0)
        xs, ys = make_positions(nl, "spread", seed=77)
        ctx.eval(t(xs), t(ys), nl.bin_w, 1.0)
        xo = x.copy()
        xo[::10] = nl.xh + 100.0
        ctx.eval(t(xo), t(y), nl.bin_w, 1.0)
        ctx.density_grad(t(xs), t(ys))
        hx = [torch.as_tensor(a).pin_memory() for a in (x, x1, xs)]
        hy = [torch.as_tensor(a).pin_memory() for a in (y, y1, ys)]
        hg = [(torch.zeros(nl.num_cells).pin_memory(), torch.zeros(nl.num_cells).pin_memory()) for _ in hx]
        hs = torch.zeros(4, dtype=torch.float64).pin_memory()
        for k in range(3):
            dp.dp_eval_host_async(ctx, hx[k], hy[k], nl.bin_w, 1.0, hg[k][0], hg[k][1], hs, True)
        dp.dp_eval_host_wait(ctx)
        dp.dp_debug_sort_stats(ctx)
        torch.cuda.synchronize()
        ctx.close()
os.environ["DP_FFT"] = "1"
m = 256
nlm = custom_netlist([0], [], [], [], [1.0], [1.0], (0, 0, 10.0 * m, 10.0 * m), (m, m))
cm = dp.dp_create(nlm)
rho = t(np.random.default_rng(0).random((m, m)))
cm.fields(rho)
dp.dp_debug_sharded_fields(cm, 4, rho)
torch.cuda.synchronize()
print("sanitize workload done")
