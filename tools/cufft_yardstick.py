"""Yardstick for the field passes: cuFFT (via torch.fft) 2-D transforms of the bigblue4 map size,
CUDA-graph device time per call (not used by the product path)."""
import json
import torch

dev = torch.device("cuda", 0)
out = {}
for n in (512, 1024, 2048):
    z = torch.randn(n, n, dtype=torch.complex64, device=dev)
    r = torch.randn(n, n, dtype=torch.float32, device=dev)
    cases = {"c2c_fft2": lambda: torch.fft.fft2(z), "r2c_rfft2": lambda: torch.fft.rfft2(r),
             "c2c_fft_rows": lambda: torch.fft.fft(z, dim=1)}
    for name, fn in cases.items():
        for _ in range(5):
            fn()
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            for _ in range(20):
                fn()
        g.replay()
        torch.cuda.synchronize()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        for _ in range(10):
            g.replay()
        b.record()
        torch.cuda.synchronize()
        out[f"{name}_{n}_us"] = a.elapsed_time(b) / 200 * 1e3
print(json.dumps(out))
