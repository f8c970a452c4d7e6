"""Shared helpers for the parity tests (tolerances are stated here, once).

Tolerance semantics (DESIGN.md §Readings A12; north_star: "max relative error 1e-4 for
the fp32 path and 2e-2 (abs 1e-2) for the bf16 tensor-core path"), elementwise per output
tensor X against the fp64 oracle R:
    fp32 : |X - R| <= 1e-4 * |R| + 1e-4 * max|R|
           (a tensor whose exact value is identically 0 -- dq = dk = 0 when w = 0 or every
            window holds one key -- gets the absolute bound 1e-5 instead: fp32 rounding of
            P (dP - D) leaves ~1e-7-level residues there and a relative bound would be 0)
    bf16 : |X - R| <= 2e-2 * |R| + 1e-2
"""
from __future__ import annotations

import numpy as np

TOL = {"f32": (1e-4, 1e-4, True), "bf16": (2e-2, 1e-2, False)}


def compare(name: str, got, ref, dtype: str):
    got = np.asarray(got, dtype=np.float64)
    ref = np.asarray(ref, dtype=np.float64)
    assert got.shape == ref.shape, (name, got.shape, ref.shape)
    rtol, atol, atol_rel_to_max = TOL[dtype]
    scale = np.abs(ref).max() if ref.size else 0.0
    if atol_rel_to_max:
        atol_eff = atol * scale if scale > 0 else 1e-5
    else:
        atol_eff = atol
    err = np.abs(got - ref)
    bound = atol_eff + rtol * np.abs(ref)
    bad = ~(err <= bound)   # also catches NaN
    if bad.any():
        idx = np.unravel_index(np.argmax(np.where(bad, err - bound, -np.inf)), err.shape)
        raise AssertionError(
            f"{name} [{dtype}]: {bad.sum()} / {err.size} elements out of tolerance; worst at "
            f"{idx}: got {got[idx]!r} ref {ref[idx]!r} (err {err[idx]:.3e} > {bound[idx]:.3e}); "
            f"max abs err {np.nanmax(err):.3e}, max|ref| {scale:.3e}")
    return float(err.max()) if err.size else 0.0
