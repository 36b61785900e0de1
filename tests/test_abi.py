"""C-ABI checks that need no GPU: the library builds/loads, exports every symbol that
include/dp.h declares, validates arguments before touching the device, reports errors through
dp_last_error, and computes the host-only partition plan."""
import ctypes
import os
import re
import subprocess

import numpy as np
import pytest

import paper_conf_dac_lindlrkp19_b200 as dp
from synth import custom_netlist, make_netlist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "dp.h")


@pytest.fixture(scope="module")
def L():
    dp.build()
    return dp.lib()


def header_functions():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(dp_[a-z0-9_]+)\s*\(", src)))


def test_header_symbols_exported(L):
    declared = header_functions()
    assert len(declared) >= 15
    out = subprocess.run(["nm", "-D", "--defined-only", dp.LIB], capture_output=True, text=True, check=True).stdout
    exported = set(re.findall(r"\bT (dp_[a-z0-9_]+)\b", out))
    missing = [f for f in declared if f not in exported]
    assert not missing, f"declared in dp.h but not exported: {missing}"
    assert sorted(dp.EXPORTED_SYMBOLS) == declared
    for f in declared:
        assert hasattr(L, f)


def test_library_is_sm100a(L):
    out = subprocess.run(["cuobjdump", "--list-elf", dp.LIB], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_version_and_error_string(L):
    assert L.dp_version() >= 100
    assert isinstance(L.dp_last_error(), bytes)


def _structs(nl, bins=None, stretch=1):
    s, keep = dp._netlist_struct(nl)
    g = dp._grid_struct(nl, stretch)
    if bins:
        g.bins_x, g.bins_y = bins
    return s, g, keep


def _create_status(L, s, g):
    h = ctypes.c_void_p()
    return L.dp_create(ctypes.byref(s), ctypes.byref(g), 0, ctypes.byref(h))


def test_validation_before_device(L):
    nl = make_netlist("tiny")
    # bad CSR
    bad = make_netlist("tiny")
    bad.net_start = bad.net_start.copy()
    bad.net_start[5] = bad.net_start[6] + 1
    s, g, keep = _structs(bad)
    assert _create_status(L, s, g) == 1 and b"nondecreasing" in L.dp_last_error()
    bad = make_netlist("tiny")
    bad.pin2cell = bad.pin2cell.copy()
    bad.pin2cell[3] = bad.num_cells
    s, g, keep = _structs(bad)
    assert _create_status(L, s, g) == 1 and b"pin2cell" in L.dp_last_error()
    bad = make_netlist("tiny")
    bad.cell_w = bad.cell_w.copy()
    bad.cell_w[0] = -1
    s, g, keep = _structs(bad)
    assert _create_status(L, s, g) == 1
    # unsupported bins
    s, g, keep = _structs(nl, bins=(48, 64))
    assert _create_status(L, s, g) == 2
    s, g, keep = _structs(nl, bins=(8, 8))
    assert _create_status(L, s, g) == 2
    s, g, keep = _structs(nl, stretch=2)
    assert _create_status(L, s, g) == 1
    # NULL
    h = ctypes.c_void_p()
    assert L.dp_create(None, None, 0, ctypes.byref(h)) == 1


def test_no_cpu_fallback_without_gpu(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    nl = make_netlist("tiny")
    s, g, keep = _structs(nl)
    assert _create_status(L, s, g) == 4  # DP_ERR_CUDA: no device, no CPU path
    with pytest.raises(dp.DPError, match="CUDA"):
        dp.dp_create(nl)


def test_eval_null_ctx(L):
    st = L.dp_eval(None, None, None, 1.0, 1.0, None, None, None, None, None, None, None)
    assert st == 1


@pytest.mark.parametrize("world", [1, 2, 3, 8])
def test_partition_plan(world):
    """Cells: world contiguous blocks of ceil(N / world).  Nets (net-partitioned WA, DESIGN.md
    §6): every net of degree >= 2 is evaluated and counted on exactly one rank, nets of degree
    0 / 1 on none."""
    nl = make_netlist("tiny")
    owners = np.zeros(nl.num_nets, dtype=int)
    covered = np.zeros(nl.num_cells, dtype=int)
    B = -(-nl.num_cells // world)
    for r in range(world):
        cb, ce, mask = dp.dp_partition_plan(nl, r, world)
        assert (cb, ce) == (min(nl.num_cells, r * B), min(nl.num_cells, (r + 1) * B))
        covered[cb:ce] += 1
        assert set(np.unique(mask)) <= {0, 3}
        owners += mask == 3
    assert np.all(covered == 1)
    deg = nl.degrees()
    assert np.all(owners[deg >= 2] == 1) and np.all(owners[deg < 2] == 0)


@pytest.fixture(scope="module")
def adaptec1():
    return make_netlist("adaptec1")


@pytest.mark.parametrize("world", [2, 4, 8])
def test_partition_balance(adaptec1, world):
    """The WA work of the busiest rank: at most 1.2 / world of the pins (VERDICT r1 target; the
    owner-computes partition of round 1 evaluated 2.07 N_p in total at 8 ranks, 0.26 N_p on the
    busiest)."""
    nl = adaptec1
    deg = nl.degrees()
    pins = [int(deg[dp.dp_partition_plan(nl, r, world)[2] == 3].sum()) for r in range(world)]
    assert sum(pins) == int(deg[deg >= 2].sum())
    assert max(pins) <= 1.2 * sum(pins) / world, pins
