"""Device time of the evaluation's parts in isolation (bigblue4): the density chain alone
(dp_density_grad), the WA part alone (dp_wl_grad), the full dp_eval — each as back-to-back calls
(the library's own captured graph per call) — to see what the overlap and the kernel boundaries
cost.  One JSON line."""
import json
import sys

import torch

sys.path.insert(0, ".")
import paper_conf_dac_lindlrkp19_b200 as dp  # noqa: E402
from synth import make_netlist, make_positions  # noqa: E402

dev = torch.device("cuda", 0)
nl = make_netlist(sys.argv[1] if len(sys.argv) > 1 else "bigblue4")
x, y = make_positions(nl)
xt, yt = torch.as_tensor(x, device=dev), torch.as_tensor(y, device=dev)
ctx = dp.dp_create(nl)
gx = torch.empty(nl.num_cells, device=dev)
gy = torch.empty_like(gx)
sc = torch.zeros(4, dtype=torch.float64, device=dev)
s = torch.cuda.current_stream()


def timed(fn, n=300):
    for _ in range(20):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3


out = {"eval_us": timed(lambda: dp.dp_eval(ctx, xt, yt, nl.bin_w, 1.0, gx, gy, sc[0:1], sc[1:2], sc[2:3], None, s)),
       "density_only_us": timed(lambda: dp.dp_density_grad(ctx, xt, yt, gx, gy, sc[2:3], s)),
       "wa_only_us": timed(lambda: dp.dp_wl_grad(ctx, xt, yt, nl.bin_w, gx, gy, sc[1:2], s))}
dp.dp_profile_enable(ctx, True)
timed(lambda: dp.dp_density_grad(ctx, xt, yt, gx, gy, sc[2:3], s), 100)
dp.dp_profile_enable(ctx, False)
st, n = dp.dp_profile_read(ctx)
out["density_only_stages_us"] = {k: v / max(n, 1) * 1e3 for k, v in st.items()}
print(json.dumps(out))
