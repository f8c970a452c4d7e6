"""GPU parity of SubdivNet's circular difference (include/ft_subdiv.h, csrc/subdiv.cu) against the
fp64 oracle (oracle/subdiv.py) on the same seeded inputs: ordered and shuffled closed torus meshes,
the vector (16-byte) and scalar kernels, fp32 and bf16 storage, and a full-size mesh."""
from __future__ import annotations

import numpy as np
import pytest
import torch

from _util import compare
from oracle import subdiv as osd
from synth import mesh_features, torus_mesh

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def sd():
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    import paper_conf_pldi_tangzwjzyz22_b200 as ft
    from paper_conf_pldi_tangzwjzyz22_b200 import subdiv

    ft.load_library(build_if_missing=True)
    return subdiv


def _run(sd, nx, ny, f, dtype, shuffle, seed=0, symmetric=False):
    adj = torus_mesh(nx, ny, shuffle)
    x = mesh_features(adj.shape[0], f, seed, dtype)
    dev = torch.device("cuda:0")
    e, dy = x["e"].to(dev), x["dy"].to(dev)
    a = torch.from_numpy(adj.astype(np.int32)).to(dev)
    y = sd.circdiff_fwd(e, a)
    de = sd.circdiff_bwd(e, a, dy, symmetric=symmetric)
    torch.cuda.synchronize()
    compare("y", y.double().cpu().numpy(), osd.fwd(x["e64"], adj), dtype)
    compare("de", de.double().cpu().numpy(), osd.bwd(x["e64"], adj, x["dy64"]), dtype)


@pytest.mark.parametrize("f", [13, 64, 128, 8, 4])
@pytest.mark.parametrize("dtype", ["f32", "bf16"])
@pytest.mark.parametrize("shuffle", [None, 3])
@pytest.mark.parametrize("symmetric", [False, True])
def test_circdiff_parity(sd, f, dtype, shuffle, symmetric):
    _run(sd, 40, 30, f, dtype, shuffle, symmetric=symmetric)


def test_circdiff_tiny_and_full_size(sd):
    _run(sd, 2, 2, 3, "f32", None)                      # 8 faces
    _run(sd, 1024, 1024, 64, "bf16", None, seed=1)      # 2M faces, bench size
    _run(sd, 1024, 1024, 64, "f32", None, seed=1, symmetric=True)
    _run(sd, 512, 512, 64, "f32", 5, seed=2)            # shuffled, 512K faces


def test_circdiff_gather_is_deterministic(sd):
    adj = torus_mesh(64, 64, 2)
    x = mesh_features(adj.shape[0], 32, 6, "f32")
    dev = torch.device("cuda:0")
    e, dy = x["e"].to(dev), x["dy"].to(dev)
    a = torch.from_numpy(adj.astype(np.int32)).to(dev)
    r = [sd.circdiff_bwd(e, a, dy, symmetric=True) for _ in range(3)]
    assert all(torch.equal(r[0], t) for t in r[1:])


def test_circdiff_autograd(sd):
    adj = torus_mesh(10, 12, 1)
    x = mesh_features(adj.shape[0], 16, 4, "f32")
    dev = torch.device("cuda:0")
    e = x["e"].to(dev).requires_grad_(True)
    a = torch.from_numpy(adj.astype(np.int32)).to(dev)
    y = sd.circdiff(e, a)
    (y * x["dy"].to(dev)).sum().backward()
    compare("de", e.grad.double().cpu().numpy(), osd.bwd(x["e64"], adj, x["dy64"]), "f32")
