"""Locate density-gradient discrepancies at bigblue4 scale: per-cell error vs the oracle split by
small / large cells, and the bin-map error."""
import sys

import numpy as np
import torch

sys.path.insert(0, '.')
import oracle  # noqa: E402
import paper_conf_dac_lindlrkp19_b200 as dp  # noqa: E402
from synth import make_netlist, make_positions  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else 'bigblue4'
nl = make_netlist(name)
x, y = make_positions(nl)
ctx = dp.dp_create(nl)
xt, yt = torch.as_tensor(x, device='cuda'), torch.as_tensor(y, device='cuda')
out = ctx.density_grad(xt, yt)
rho_g = ctx.density_map(xt, yt).cpu().numpy().astype(np.float64)
D, gx, gy, parts = oracle.density(nl, x, y, 1)
print('D rel', abs(out['energy'].item() - D) / D)
print('rho max abs err', np.abs(rho_g - parts['rho']).max(), 'max rho', parts['rho'].max())
b = nl.bin_w
large = (nl.cell_w > 2 * b) | (nl.cell_h > 2 * b)
for k, ref in (('gx', gx), ('gy', gy)):
    g = out[k].cpu().numpy().astype(np.float64)
    rms = np.sqrt(np.mean(ref ** 2))
    ratio = np.abs(g - ref) / (1e-3 * np.maximum(np.abs(ref), 1e-2 * rms))
    for lab, m in (('small', ~large), ('large', large)):
        i = np.argmax(np.where(m, ratio, -1))
        print(k, lab, 'n', m.sum(), 'worst ratio %.3f' % ratio[i], 'idx', i, 'got', g[i], 'ref', ref[i],
              'w,h', nl.cell_w[i], nl.cell_h[i], 'x,y', x[i], y[i])
    bad = np.nonzero(ratio > 1)[0]
    print(k, 'n bad', len(bad), 'first', bad[:10])
