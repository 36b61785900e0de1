"""A/B of the field transforms as dense DCT-matrix GEMMs on the tensor cores (cuBLAS bf16 -> fp32,
the 3-term bf16 split X Y ~ Xh Yh + Xh Yl + Xl Yh) against libdp's FFT field passes, at 512^2 and
1024^2.  The GEMM path is the full solve: a = C rho C^T (2 GEMMs),
A_X, A_Y by the spectral scaling, xi_X = S' A_X C'^T and xi_Y = C' A_Y S'^T (4 GEMMs); each GEMM
as 3 bf16 products with fp32 accumulation and output.  cuBLAS stands in for the best a
hand-written tcgen05 GEMM could do.  Prints one JSON line per size."""
import json
import math
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
import paper_conf_dac_lindlrkp19_b200 as dp  # noqa: E402
from synth import custom_netlist  # noqa: E402

dev = torch.device("cuda", 0)


def mats(n, length):
    t = np.arange(n)
    u = np.arange(n)
    ang = np.pi * np.outer(u, t + 0.5) / n                     # [u][t]
    C = (2.0 / n) * np.cos(ang)                               # forward DCT (eq 7a x 2/N)
    ci = np.cos(ang.T).copy()                                 # inverse IDCT (eq 7b): [t][u]
    ci[:, 0] *= 0.5
    si = np.sin(ang.T)                                        # IDXST (eq 8a): [t][u]
    k = np.pi * u / length
    return C, ci, si, k


def ref_fields(rho, C, ci, si, k):
    a = C @ rho @ C.T
    k2 = k[:, None] ** 2 + k[None, :] ** 2
    inv = np.zeros_like(k2)
    inv[k2 > 0] = 1.0 / k2[k2 > 0]
    ax, ay = a * k[:, None] * inv, a * k[None, :] * inv
    return si @ ax @ ci.T, ci @ ay @ si.T


def split(m, terms=2):
    t = torch.as_tensor(m, dtype=torch.float64, device=dev)
    out = []
    for _ in range(terms):
        h = t.to(torch.bfloat16)
        out.append(h)
        t = t - h.double()
    return tuple(out)


def mm3(a, b):
    """Products of bf16 split terms with fp32 accumulation / output: 2-term splits -> the 3
    products of order <= 1 (h h, h l, l h); 3-term splits -> the 6 products of order <= 2."""
    out = None
    for i, ai in enumerate(a):
        for j, bj in enumerate(b):
            if i + j < len(a):
                p = torch.mm(ai, bj, out_dtype=torch.float32)
                out = p if out is None else out + p
    return out


TERMS = 2


def split32(x):
    out = []
    for _ in range(TERMS):
        h = x.to(torch.bfloat16)
        out.append(h)
        x = x - h.float()
    return tuple(out)


def gemm_fields(rho, C, CT, ci, ciT, si, siT, kx, ky):
    a = mm3(split32(mm3(C, split32(rho))), CT)
    k2 = kx[:, None] ** 2 + ky[None, :] ** 2
    inv = torch.where(k2 > 0, 1.0 / torch.where(k2 > 0, k2, torch.ones_like(k2)), torch.zeros_like(k2))
    ax, ay = a * kx[:, None] * inv, a * ky[None, :] * inv
    xx = mm3(split32(mm3(si, split32(ax))), ciT)
    xy = mm3(split32(mm3(ci, split32(ay))), siT)
    return xx, xy


def timed(fn, n=50):
    """Device time per call of fn captured in a CUDA graph (no host launch overhead)."""
    s = torch.cuda.Stream()
    s.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(s):
        for _ in range(3):
            fn()
    torch.cuda.current_stream().wait_stream(s)
    torch.cuda.synchronize()
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        fn()
    for _ in range(3):
        g.replay()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n):
        g.replay()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n * 1e3


for n, TERMS in ((512, 2), (1024, 2), (512, 3), (1024, 3)):
    L = 36.0 * n
    C, ci, si, k = mats(n, L)
    rho = np.random.default_rng(n).random((n, n)) * 2.0
    rx, ry = ref_fields(rho, C, ci, si, k)
    Cs, CTs, cis, ciTs, sis, siTs = (split(m, TERMS) for m in (C, C.T.copy(), ci, ci.T.copy(), si, si.T.copy()))
    kt = torch.as_tensor(k, dtype=torch.float32, device=dev)
    rho_t = torch.as_tensor(rho, dtype=torch.float32, device=dev)
    gx, gy = gemm_fields(rho_t, Cs, CTs, cis, ciTs, sis, siTs, kt, kt)
    us_gemm = timed(lambda: gemm_fields(rho_t, Cs, CTs, cis, ciTs, sis, siTs, kt, kt))

    def err(g, r):
        g = g.double().cpu().numpy()
        return float(np.linalg.norm(g - r) / np.linalg.norm(r)), float(np.abs(g - r).max() / np.abs(r).max())

    nl = custom_netlist([0], [], [], [], [1.0], [1.0], (0, 0, L, L), (n, n))
    ctx = dp.dp_create(nl)
    f = ctx.fields(rho_t, want_psi=False)
    xx = torch.empty((n, n), dtype=torch.float32, device=dev)
    xy = torch.empty_like(xx)
    en = torch.zeros(1, dtype=torch.float64, device=dev)
    us_fft = timed(lambda: dp.dp_debug_fields(ctx, rho_t, None, xx, xy, en, torch.cuda.current_stream()))
    nprod = 3 if TERMS == 2 else 6
    flops = 6 * nprod * 2.0 * n ** 3
    print(json.dumps({"bins": n, "bf16_terms": TERMS, "bf16_products_per_gemm": nprod, "gemm_us": us_gemm, "gemm_tflops": flops / (us_gemm * 1e-6) / 1e12,
                      "gemm_err_xi_x": err(gx, rx), "gemm_err_xi_y": err(gy, ry),
                      "fft_fields_us": us_fft, "fft_err_xi_x": err(f["xi_x"], rx), "fft_err_xi_y": err(f["xi_y"], ry),
                      "note": "CUDA-graph device time per call; fft_fields_us = dp_debug_fields without psi (the field passes + "
                              "the split of xi into two planes + the energy finalize); gemm = 6 x products cuBLAS "
                              "bf16 GEMMs (fp32 out) + scaling; errors = (rel-L2, max/max) vs fp64"}),
          flush=True)
