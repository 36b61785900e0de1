"""Shared helpers for GPU-vs-oracle parity tests (tolerances from BASELINE.json north_star,
per-entry floor from reading A25)."""
import numpy as np

REL_SCALAR = 1e-4     # WA, D, obj: relative 1e-4
REL_L2 = 1e-4         # gradients: ||g - r|| / ||r|| <= 1e-4
REL_ENTRY = 1e-3      # gradients: per entry |g - r| <= 1e-3 max(|r|, 1e-2 rms(r))


def to_np(t):
    return t.detach().cpu().numpy().astype(np.float64)


def check_scalar(name, got, ref, rel=REL_SCALAR):
    got = float(got)
    err = abs(got - ref) / max(abs(ref), 1e-300)
    assert err <= rel, f"{name}: got {got!r} ref {ref!r} rel err {err:.3e} > {rel}"


def check_vector(name, got, ref, rel_l2=REL_L2, rel_entry=REL_ENTRY):
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    assert got.shape == ref.shape, (name, got.shape, ref.shape)
    assert np.all(np.isfinite(got)), f"{name}: non-finite entries"
    nr = np.linalg.norm(ref)
    if nr == 0:
        assert np.abs(got).max() <= 1e-6, f"{name}: expected zeros, max {np.abs(got).max()}"
        return
    l2 = np.linalg.norm(got - ref) / nr
    rms = nr / np.sqrt(ref.size)
    bound = rel_entry * np.maximum(np.abs(ref), 1e-2 * rms)
    bad = np.abs(got - ref) > bound
    worst = int(np.argmax(np.abs(got - ref) / bound))
    assert l2 <= rel_l2, f"{name}: rel L2 {l2:.3e} > {rel_l2}"
    assert not bad.any(), (f"{name}: {int(bad.sum())} entries over per-entry bound; worst idx {worst} "
                           f"got {got[worst]!r} ref {ref[worst]!r}")


def check_map(name, got, ref, rel=1e-5):
    """Maps (rho, psi, xi): max abs error relative to the map's max magnitude."""
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    scale = max(np.abs(ref).max(), 1e-300)
    err = np.abs(got - ref).max() / scale
    assert err <= rel, f"{name}: max err {err:.3e} of max |ref| {scale:.3e} > {rel}"
