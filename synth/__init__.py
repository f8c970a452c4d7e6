"""Seeded synthetic inputs for window attention — shared by tests, bench and smoke.

This module holds NO arithmetic of the method (no scores, softmax or gradients):
it only draws the random inputs and rounds them to the storage dtype.  Both the
fp64 oracle (`oracle/`) and the CUDA path (`paper_conf_pldi_tangzwjzyz22_b200`)
consume what it returns; neither imports the other.

Recipe:
  * numpy ``Generator(PCG64(seed))`` draws q, k, v, dout in that order, each
    i.i.d. U(-1, 1) in fp64, shape [B, H, L, d] ("We use random
    input for the test").
  * The draws are rounded to the storage dtype (fp32 by numpy, bf16 by torch's
    round-to-nearest-even), and the oracle reads the ROUNDED values upcast
    exactly to fp64, so parity measures kernel error, not input quantisation.
  * ``q_scale`` multiplies q before rounding (the x16 "overflow probe").
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

__all__ = ["WinAttnShape", "CONFIGS", "make_inputs", "round_to", "TORCH_DTYPES"]


@dataclass(frozen=True)
class WinAttnShape:
    batch: int
    heads: int
    seq_len: int
    d: int
    w: int
    dilation: int = 1

    @property
    def units(self) -> int:
        return self.batch * self.heads

    @property
    def rows(self) -> int:
        return self.batch * self.heads * self.seq_len


# Named configurations (BASELINE.json "configs").
CONFIGS = {
    # configs[0]: tiny, oracle fwd+bwd + finite differences in seconds.
    "C1": WinAttnShape(1, 1, 64, 16, 4, 1),
    # configs[1]/[2]: Longformer-shaped, reading A14(a) of the FreeTensor artefact
    # (n_heads=8, seq_len=10000, feat_len=512, w=32).
    "C2a": WinAttnShape(1, 8, 10000, 512, 32, 1),
    # the artefact's dilated heads (heads 0-1 use dilation 4), run as its own call.
    "C2a_dil": WinAttnShape(1, 2, 10000, 512, 32, 4),
    # Longformer-base shape, reading A14(b).
    "C2b": WinAttnShape(1, 12, 4096, 64, 256, 1),
    # configs[3]: dilated, large window, 16K tokens.
    "C4d2": WinAttnShape(1, 12, 16384, 64, 256, 2),
    "C4d4": WinAttnShape(1, 12, 16384, 64, 256, 4),
    # configs[4]: sweep corners (H in {8..64}, L in {4K..32K}, w in {32, 256}).
    "C5_small_w32": WinAttnShape(1, 8, 4096, 64, 32, 1),
    "C5_big_w32": WinAttnShape(1, 64, 32768, 64, 32, 1),
    "C5_big_w256": WinAttnShape(1, 64, 32768, 64, 256, 1),
    # one unit of 2^21 rows: 21-bit row indices, 16384 tiles in one (unit, residue) problem
    "long_2M": WinAttnShape(1, 1, 2097152, 64, 32, 3),
}


def _torch():
    import torch  # local import: the oracle tests must not need CUDA

    return torch


TORCH_DTYPES = ("f32", "bf16")


def round_to(x: np.ndarray, dtype: str):
    """Round fp64 ``x`` to the storage dtype.

    Returns ``(torch_tensor_in_dtype, fp64_numpy_of_the_rounded_values)``.
    The fp64 copy is exact (both f32 and bf16 embed in fp64).
    """
    torch = _torch()
    t64 = torch.from_numpy(np.ascontiguousarray(x))
    if dtype == "f32":
        t = t64.to(torch.float32)
    elif dtype == "bf16":
        t = t64.to(torch.bfloat16)  # round-to-nearest-even
    else:
        raise ValueError(f"unknown dtype {dtype!r}")
    return t.contiguous(), t.to(torch.float64).numpy()


def make_inputs(shape: WinAttnShape, seed: int, dtype: str = "f32", q_scale: float = 1.0,
                with_dout: bool = True):
    """Draw q, k, v (and dout) for ``shape``.

    Returns a dict with torch tensors (CPU, storage dtype) under 'q','k','v','dout'
    and their exact fp64 numpy copies under 'q64','k64','v64','dout64'.
    """
    rng = np.random.Generator(np.random.PCG64(seed))
    dims = (shape.batch, shape.heads, shape.seq_len, shape.d)
    out = {}
    names = ["q", "k", "v"] + (["dout"] if with_dout else [])
    for name in names:
        x = rng.uniform(-1.0, 1.0, size=dims)
        if name == "q" and q_scale != 1.0:
            x = x * q_scale
        t, x64 = round_to(x, dtype)
        out[name] = t
        out[name + "64"] = x64
    return out


# --------------------------------------------------------------------------- SubdivNet meshes
def torus_mesh(nx: int, ny: int, shuffle_seed: int | None = None) -> np.ndarray:
    """Face adjacency [2*nx*ny, 3] (int64) of a closed triangulated torus: an nx x ny grid of
    quads, each split into two triangles, wrapping in both directions, so every face has exactly
    three edge-adjacent faces -- the manifold meshes SubdivNet convolves over (PAPER.md
    Section 2.2).  Triangle A of cell (x, y) borders B of the same cell, B of (x, y-1) and
    B of (x-1, y); triangle B borders A of the same cell, A of (x, y+1) and A of (x+1, y).
    With shuffle_seed, face ids are randomly permuted (an unordered mesh).  Pure data
    generation: no arithmetic of the method."""
    xs, ys = np.meshgrid(np.arange(nx), np.arange(ny), indexing="ij")
    cell = lambda x, y: ((x % nx) * ny + (y % ny))  # noqa: E731
    A = 2 * cell(xs, ys)
    B = A + 1
    adjA = np.stack([2 * cell(xs, ys) + 1, 2 * cell(xs, ys - 1) + 1, 2 * cell(xs - 1, ys) + 1], -1)
    adjB = np.stack([2 * cell(xs, ys), 2 * cell(xs, ys + 1), 2 * cell(xs + 1, ys)], -1)
    adj = np.empty((2 * nx * ny, 3), dtype=np.int64)
    adj[A.reshape(-1)] = adjA.reshape(-1, 3)
    adj[B.reshape(-1)] = adjB.reshape(-1, 3)
    if shuffle_seed is not None:
        perm = np.random.Generator(np.random.PCG64(shuffle_seed)).permutation(adj.shape[0])
        inv = np.empty_like(perm)
        inv[perm] = np.arange(perm.size)
        adj = inv[adj[perm]]          # new face f = old face perm[f]
    return adj


def mesh_features(n_faces: int, n_feats: int, seed: int, dtype: str = "f32"):
    """e and dy, i.i.d. U(-1, 1) drawn with PCG64(seed) in that order, rounded to the storage dtype;
    returns dict with torch tensors 'e', 'dy' and their exact fp64 numpy copies 'e64', 'dy64'."""
    rng = np.random.Generator(np.random.PCG64(seed))
    out = {}
    for name in ("e", "dy"):
        x = rng.uniform(-1.0, 1.0, size=(n_faces, n_feats))
        t, x64 = round_to(x, dtype)
        out[name] = t
        out[name + "64"] = x64
    return out
