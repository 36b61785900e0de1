"""PCIe copy rates on the box (the e2e path's bound): pinned H2D alone, D2H alone, both at once."""
import torch
n = 2_180_000 * 2   # x | y of bigblue4 (17.4 MB)
h_in = torch.empty(n).pin_memory(); h_out = torch.empty(n).pin_memory()
d_in = torch.empty(n, device="cuda"); d_out = torch.empty(n, device="cuda")
s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
def rate(fn, reps=50):
    torch.cuda.synchronize(); a = torch.cuda.Event(enable_timing=True); b = torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(reps): fn()
    torch.cuda.current_stream().wait_stream(s1); torch.cuda.current_stream().wait_stream(s2)
    b.record(); torch.cuda.synchronize()
    return reps * n * 4 / (a.elapsed_time(b) * 1e-3) / 1e9
def h2d():
    with torch.cuda.stream(s1): d_in.copy_(h_in, non_blocking=True)
def d2h():
    with torch.cuda.stream(s2): h_out.copy_(d_out, non_blocking=True)
def both():
    h2d(); d2h()
print(f"H2D alone {rate(h2d):.1f} GB/s, D2H alone {rate(d2h):.1f} GB/s, both at once {rate(both):.1f} GB/s each way")
