"""Multi-process check of the distributed partition on CPU.

gloo ranks each take libdp's host-only partition plan (dp_partition_plan), evaluate their shard
with the fp64 oracle exactly as a distributed context does (WA over the rank's own nets with a
gradient over all cells, the density map of the rank's cell block), combine with the
collectives the GPU path uses (gradient sum = reduce-scatter, bin-map sum, WA partial sum, HPWL
terms) and must reproduce the single-process oracle."""
import math
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _shard_eval(nl, x, y, gamma, cb, ce, mask):
    import oracle
    from synth import custom_netlist
    # WA over the nets this rank evaluates (mask 3, each net on one rank); gradient on every cell
    sel = np.nonzero(mask == 3)[0]
    starts = nl.net_start
    deg = starts[sel + 1] - starts[sel]
    ns = np.concatenate([[0], np.cumsum(deg)])
    pins = np.concatenate([np.arange(starts[e], starts[e + 1]) for e in sel]) if len(sel) else np.zeros(0, int)
    sub = custom_netlist(ns, nl.pin2cell[pins], nl.pin_dx[pins], nl.pin_dy[pins], nl.cell_w, nl.cell_h,
                         (nl.xl, nl.yl, nl.xh, nl.yh), (nl.bins_x, nl.bins_y))
    _, gx, gy, wl_net = oracle.wa(sub, x, y, gamma, per_net=True)
    wl = float(np.sum(wl_net))
    h = oracle.hpwl_nets(sub, x, y)
    # density: this rank's cells only
    cells = custom_netlist([0], [], [], [], nl.cell_w[cb:ce], nl.cell_h[cb:ce], (nl.xl, nl.yl, nl.xh, nl.yh),
                           (nl.bins_x, nl.bins_y))
    rho = oracle.density_map(cells, x[cb:ce], y[cb:ce], 1)
    return wl, gx, gy, h, rho, cells


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    import paper_conf_dac_lindlrkp19_b200 as dp
    from synth import make_netlist, make_positions
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    gamma = 7.0
    cb, ce, mask = dp.dp_partition_plan(nl, rank, world)
    wl, gx, gy, h, rho, cells = _shard_eval(nl, x, y, gamma, cb, ce, mask)
    t = torch.tensor([wl], dtype=torch.float64)
    dist.all_reduce(t)                                   # WA partial sums (fp64 all-reduce)
    rho_t = torch.from_numpy(rho.copy())
    dist.all_reduce(rho_t)                               # bin map (the GPU path sums int64)
    g = torch.from_numpy(np.stack([gx, gy]))
    dist.all_reduce(g)                                   # partial gradients of disjoint net sets (reduce-scatter)
    hs = [None] * world
    dist.all_gather_object(hs, h.tolist())
    # replicated Poisson solve on the summed map, force for own cells
    rho_full = rho_t.numpy()
    psi, xi_x, xi_y = oracle.fields(nl, oracle.dct2(rho_full))
    D = oracle.energy(nl, rho_full, psi)
    fx, fy = oracle.density_grad(cells, x[cb:ce], y[cb:ce], xi_x, xi_y, 1)
    f = torch.zeros(2, nl.num_cells, dtype=torch.float64)
    f[0, cb:ce] = torch.from_numpy(fx)
    f[1, cb:ce] = torch.from_numpy(fy)
    dist.all_reduce(f)
    if rank == 0:
        q.put(dict(wl=t.item(), gx=g[0].numpy(), gy=g[1].numpy(), hpwl=math.fsum(sum(hs, [])), D=D,
                   fx=f[0].numpy(), fy=f[1].numpy(), rho=rho_full))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_net_partitioned_shards_reassemble_the_oracle(world):
    import oracle
    from synth import make_netlist, make_positions
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    nl = make_netlist("tiny")
    x, y = make_positions(nl)
    wl, gx, gy = oracle.wa(nl, x, y, 7.0)
    assert res["wl"] == pytest.approx(wl, rel=1e-12)
    np.testing.assert_allclose(res["gx"], gx, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(res["gy"], gy, rtol=1e-12, atol=1e-12)
    assert res["hpwl"] == oracle.hpwl(nl, x, y)
    D, fx, fy, parts = oracle.density(nl, x, y, 1)
    np.testing.assert_allclose(res["rho"], parts["rho"], rtol=1e-12, atol=1e-12)
    assert res["D"] == pytest.approx(D, rel=1e-12)
    np.testing.assert_allclose(res["fx"], fx, rtol=1e-10, atol=1e-9 * np.abs(fx).max())
    np.testing.assert_allclose(res["fy"], fy, rtol=1e-10, atol=1e-9 * np.abs(fy).max())


def _sharded_poisson_worker(rank, world, port, q):
    """One rank of the row-sharded Poisson solve in fp64 with the oracle's naive
    transforms and gloo collectives: reduce-scatter of the map by row blocks, DCT over y of the
    rank's rows, all-to-all, DCT over x of its columns with the spectral scaling (A12, A15) and
    the Parseval energy partial (A8), inverse x transforms, all-to-all back, inverse y
    transforms of its rows, all-gather of the field rows."""
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import oracle
    from synth import custom_netlist, make_netlist, make_positions
    nl = make_netlist("tiny", bins=64)
    x, y = make_positions(nl)
    M = nl.bins_x
    R = C = M // world
    # this rank's cell block (the density partition) -> partial map -> "reduce-scatter"
    B = -(-nl.num_cells // world)
    cb, ce = min(nl.num_cells, rank * B), min(nl.num_cells, (rank + 1) * B)
    cells = custom_netlist([0], [], [], [], nl.cell_w[cb:ce], nl.cell_h[cb:ce], (nl.xl, nl.yl, nl.xh, nl.yh),
                           (M, M))
    rho = torch.from_numpy(oracle.density_map(cells, x[cb:ce], y[cb:ce], 1))
    dist.all_reduce(rho)
    rows = rho.numpy()[rank * R:(rank + 1) * R]                        # [R, M]

    def all_to_all(blocks):   # blocks[q] goes to rank q; returns the blocks received from each rank
        t = torch.from_numpy(np.stack(blocks))
        got = [torch.empty_like(t) for _ in range(world)]
        dist.all_gather(got, t)
        return [got[p][rank].numpy() for p in range(world)]

    t_rows = oracle.transform(oracle.DCT, rows, 1)                     # P1: DCT over y
    t_cols = np.concatenate(all_to_all([t_rows[:, qq * C:(qq + 1) * C] for qq in range(world)]), axis=0)   # [M, C]
    a = oracle.transform(oracle.DCT, t_cols, 0)                       # P2: DCT over x
    ku, kv = oracle.wavenumbers(nl)
    kvc = kv[rank * C:(rank + 1) * C]
    k2 = ku[:, None] ** 2 + kvc[None, :] ** 2
    inv = np.zeros_like(k2)
    inv[k2 > 0] = 1.0 / k2[k2 > 0]
    wu = np.where(np.arange(M) == 0, M / 4, M / 2)
    wv = np.where(np.arange(rank * C, (rank + 1) * C) == 0, M / 4, M / 2)
    e = torch.tensor([0.5 * nl.bin_w * nl.bin_h * float(np.sum(wu[:, None] * wv[None, :] * a * a * inv))],
                     dtype=torch.float64)
    dist.all_reduce(e)
    sx = oracle.transform(oracle.IDXST, a * ku[:, None] * inv, 0)
    sy = oracle.transform(oracle.IDCT, a * kvc[None, :] * inv, 0)
    s_back = all_to_all([np.stack([sx[qq * R:(qq + 1) * R], sy[qq * R:(qq + 1) * R]]) for qq in range(world)])
    sx_rows = np.concatenate([b[0] for b in s_back], axis=1)            # [R, M]
    sy_rows = np.concatenate([b[1] for b in s_back], axis=1)
    xi = torch.from_numpy(np.stack([oracle.transform(oracle.IDCT, sx_rows, 1),
                                    oracle.transform(oracle.IDXST, sy_rows, 1)]))   # P3
    got = [torch.empty_like(xi) for _ in range(world)]
    dist.all_gather(got, xi)                                            # field rows -> every rank
    if rank == 0:
        q.put(dict(xi_x=np.concatenate([g[0].numpy() for g in got]), xi_y=np.concatenate([g[1].numpy() for g in got]),
                   D=e.item()))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [4])
def test_row_sharded_poisson_reassembles_the_oracle(world):
    import oracle
    from synth import make_netlist, make_positions
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sharded_poisson_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = q.get(timeout=300)
    for p in procs:
        p.join(timeout=300)
        assert p.exitcode == 0
    nl = make_netlist("tiny", bins=64)
    x, y = make_positions(nl)
    D, _, _, parts = oracle.density(nl, x, y, 1)
    np.testing.assert_allclose(res["xi_x"], parts["xi_x"], rtol=0, atol=1e-12 * np.abs(parts["xi_x"]).max())
    np.testing.assert_allclose(res["xi_y"], parts["xi_y"], rtol=0, atol=1e-12 * np.abs(parts["xi_y"]).max())
    assert res["D"] == pytest.approx(D, rel=1e-12)   # Parseval (A8) over sharded column blocks
