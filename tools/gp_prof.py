"""Short GP run on bigblue4 (initial placement) for an ncu launch list of one iteration's kernels."""
import sys
import torch
sys.path.insert(0, ".")
import paper_conf_dac_lindlrkp19_b200 as dp  # noqa: E402
from synth import make_netlist, make_positions  # noqa: E402

nl = make_netlist(sys.argv[1] if len(sys.argv) > 1 else "bigblue4")
x, y = make_positions(nl, "initial")
dev = torch.device("cuda", 0)
ctx = dp.dp_create(nl)
loop = dp.GpLoop(ctx, max_history=64)
loop.init(torch.as_tensor(x, device=dev), torch.as_tensor(y, device=dev))
loop.run(int(sys.argv[2]) if len(sys.argv) > 2 else 20)
torch.cuda.synchronize()
a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
a.record()
loop.run(40)
b.record()
torch.cuda.synchronize()
st = dp.dp_debug_sort_stats(ctx) if hasattr(dp, "dp_debug_sort_stats") and "DP_LIB_AB" not in __import__("os").environ else {}
print("us/iteration", round(a.elapsed_time(b) / 40 * 1e3, 1), st)
