"""Launch a few cuFFT 1024-point transforms (row FFT of 1024x1024 c64, 2-D fft2) for ncu."""
import torch
z = torch.randn(1024, 1024, dtype=torch.complex64, device="cuda")
for _ in range(3):
    torch.fft.fft(z, dim=1)
    torch.fft.fft2(z)
    torch.fft.ifft(z, dim=0)
torch.cuda.synchronize()
