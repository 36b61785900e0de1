"""Repeat the 'initial'-placement density parity case and report how close it runs to the
per-entry bound (reading A25): max |g - r| / (1e-3 max(|r|, 1e-2 rms r)) over repeats."""
import sys

import numpy as np
import torch

sys.path.insert(0, '.')
import oracle  # noqa: E402
import paper_conf_dac_lindlrkp19_b200 as dp  # noqa: E402
from synth import make_netlist, make_positions  # noqa: E402

nl = make_netlist('tiny')
ctx = dp.dp_create(nl)
for dist in ('initial', 'spread'):
    x, y = make_positions(nl, dist)
    D, gx, gy, parts = oracle.density(nl, x, y, 1)
    worst = []
    for _ in range(10):
        out = ctx.density_grad(torch.as_tensor(x, device='cuda'), torch.as_tensor(y, device='cuda'))
        wr = (0, 0, 0, 0)
        for k, ref in (('gx', gx), ('gy', gy)):
            rms = np.sqrt(np.mean(ref ** 2))
            bound = 1e-3 * np.maximum(np.abs(ref), 1e-2 * rms)
            g = out[k].cpu().numpy().astype(np.float64)
            r = np.abs(g - ref) / bound
            if r.max() > wr[0]:
                wr = (r.max(), k + str(int(r.argmax())), abs(out['energy'].item() - D) / D,
                      np.linalg.norm(g - ref) / np.linalg.norm(ref))
        worst.append(wr)
    print(dist, 'per-entry ratio (1.0 = at bound):', ['%.3f' % w[0] for w in worst])
    print(dist, 'worst idx', [w[1] for w in worst][:5], 'D rel err %.2e' % max(w[2] for w in worst),
          'L2 rel %.2e' % max(w[3] for w in worst))
