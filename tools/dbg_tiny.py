import sys, os, traceback
sys.path.insert(0, ".")
import numpy as np, torch
import paper_conf_dac_lindlrkp19_b200 as dp
from synth import make_netlist, make_positions
nl = make_netlist("tiny")
print("zero-area cells", int(((nl.cell_w * nl.cell_h) == 0).sum()), "large", int(((nl.cell_w > 2*nl.bin_w)|(nl.cell_h > 2*nl.bin_h)).sum()))
x, y = make_positions(nl)
t = lambda a: torch.as_tensor(a, device="cuda")
for step in ("create", "density_map", "density_grad", "eval"):
    try:
        if step == "create": ctx = dp.dp_create(nl)
        elif step == "density_map": ctx.density_map(t(x), t(y))
        elif step == "density_grad": ctx.density_grad(t(x), t(y))
        else: ctx.eval(t(x), t(y), nl.bin_w, 1.0)
        torch.cuda.synchronize(); print("ok", step, dp.dp_debug_sort_stats(ctx) if step != "create" else "")
    except Exception as e:
        print("FAIL", step, repr(e)[:300]); break
