"""Host cost per dp_eval call vs device time (graph / no-graph): run under gpurun."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_dac_lindlrkp19_b200 as dp
from synth import make_netlist, make_positions

nl = make_netlist(sys.argv[1] if len(sys.argv) > 1 else "bigblue4")
x, y = make_positions(nl)
dev = torch.device("cuda", 0)
ctx = dp.dp_create(nl, 0)
xt, yt = torch.as_tensor(x, device=dev), torch.as_tensor(y, device=dev)
gx = torch.empty(nl.num_cells, device=dev); gy = torch.empty_like(gx)
sc = torch.zeros(4, dtype=torch.float64, device=dev)
s = torch.cuda.current_stream()
def step():
    dp.dp_eval(ctx, xt, yt, float(nl.bin_w), 1.0, gx, gy, sc[0:1], sc[1:2], sc[2:3], None, s)
for _ in range(20):
    step()
torch.cuda.synchronize()
for n in (50, 500):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    h0 = time.perf_counter(); a.record(s)
    for _ in range(n):
        step()
    h1 = time.perf_counter(); b.record(s); torch.cuda.synchronize(); h2 = time.perf_counter()
    print(f"n={n} host issue {1e6*(h1-h0)/n:.1f} us/call, device {1e3*a.elapsed_time(b)/n:.1f} us/call, wall {1e6*(h2-h0)/n:.1f}")
# pure issue cost without the GPU being busy: ctypes marshalling only
t0 = time.perf_counter()
for _ in range(200):
    dp.dp_get_info(ctx)
print(f"dp_get_info {1e6*(time.perf_counter()-t0)/200:.1f} us/call")
