"""Pins of the SubdivNet circular-difference oracle (oracle/subdiv.py) -- CPU only.

Each check is independent of the oracle's own loops: a hand-worked golden example
(tests/golden/subdiv_tetra.txt), the operator formulation of PAPER.md Fig. 2(c) written with
numpy / torch ops (index_select, cat, abs, sum) and its torch.autograd gradient, invariants
(y >= 0, invariance under rotating or reversing a face's adjacency, y = 0 for equal neighbours,
sum of de = 0) and central finite differences."""
from __future__ import annotations

import os

import numpy as np
import pytest
import torch

from oracle import subdiv as osd
from synth import mesh_features, torus_mesh

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "subdiv_tetra.txt")


def _golden():
    rec = {"adj": []}
    for line in open(GOLDEN):
        if line.startswith("#") or not line.strip():
            continue
        key, *vals = line.split()
        if key == "adj":
            rec["adj"].append([int(v) for v in vals])
        else:
            rec[key] = np.array([float(v) for v in vals])
    return np.array(rec["adj"]), rec


def test_golden_tetrahedron():
    adj, g = _golden()
    e = g["e"].reshape(-1, 1)
    np.testing.assert_array_equal(osd.fwd(e, adj)[:, 0], g["y"])
    np.testing.assert_array_equal(osd.bwd(e, adj, np.ones_like(e))[:, 0], g["de"])


def _operator_form(e, adj):
    """Fig. 2(c) with torch ops: index_select -> cat (rotate) -> abs -> sum."""
    n, f = e.shape
    adj_feat = torch.index_select(e, 0, adj.flatten()).reshape(n, 3, f)
    reordered = torch.cat([adj_feat[:, 1:], adj_feat[:, :1]], dim=1)
    return torch.sum(torch.abs(adj_feat - reordered), dim=1)


@pytest.mark.parametrize("nx,ny,f,shuffle", [(3, 4, 5, None), (8, 5, 16, 7), (2, 2, 3, 1)])
def test_matches_operator_formulation_and_autograd(nx, ny, f, shuffle):
    adj = torus_mesh(nx, ny, shuffle)
    x = mesh_features(adj.shape[0], f, 3, "f32")
    e64, dy64 = x["e64"], x["dy64"]
    et = torch.from_numpy(e64).requires_grad_(True)
    y_ref = _operator_form(et, torch.from_numpy(adj))
    (y_ref * torch.from_numpy(dy64)).sum().backward()
    np.testing.assert_allclose(osd.fwd(e64, adj), y_ref.detach().numpy(), rtol=0, atol=1e-13)
    np.testing.assert_allclose(osd.bwd(e64, adj, dy64), et.grad.numpy(), rtol=0, atol=1e-13)


def test_invariants():
    adj = torus_mesh(6, 7, 3)
    x = mesh_features(adj.shape[0], 9, 5, "f32")
    e, dy = x["e64"], x["dy64"]
    y = osd.fwd(e, adj)
    assert (y >= 0).all()
    np.testing.assert_allclose(osd.fwd(e, np.roll(adj, 1, axis=1)), y, rtol=0, atol=1e-13)
    np.testing.assert_allclose(osd.fwd(e, adj[:, ::-1].copy()), y, rtol=0, atol=1e-13)
    de = osd.bwd(e, adj, dy)
    np.testing.assert_allclose(de.sum(axis=0), 0.0, atol=1e-12)     # each pair adds +s and -s
    # equal features on all three neighbours of every face -> y = 0 and de = 0
    const = np.tile(np.arange(9.0), (adj.shape[0], 1))
    assert np.abs(osd.fwd(const, adj)).max() == 0.0
    assert np.abs(osd.bwd(const, adj, dy)).max() == 0.0             # sign(0) = 0 (reading S1)


def test_finite_differences():
    adj = torus_mesh(3, 3, 2)
    x = mesh_features(adj.shape[0], 2, 9, "f32")
    e, dy = x["e64"], x["dy64"]
    de = osd.bwd(e, adj, dy)
    h = 1e-7
    num = np.zeros_like(e)
    for idx in np.ndindex(*e.shape):
        ep, em = e.copy(), e.copy()
        ep[idx] += h
        em[idx] -= h
        num[idx] = ((osd.fwd(ep, adj) * dy).sum() - (osd.fwd(em, adj) * dy).sum()) / (2 * h)
    np.testing.assert_allclose(num, de, rtol=0, atol=1e-6)


def test_torus_mesh_is_a_closed_manifold():
    for nx, ny, sh in ((2, 2, None), (5, 3, None), (4, 6, 11)):
        adj = torus_mesh(nx, ny, sh)
        n = adj.shape[0]
        assert n == 2 * nx * ny and adj.min() >= 0 and adj.max() < n
        for f in range(n):
            assert len(set(adj[f])) == 3 and f not in adj[f]
            for g in adj[f]:
                assert f in adj[g]           # edge adjacency is symmetric
