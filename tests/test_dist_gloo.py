"""World-size-2 gloo tests (CPU) of the (batch, head) sharding host logic in dist.py.

The per-slab compute is the fp64 oracle here (the CUDA kernels need a GPU); the test
checks that scatter -> per-rank compute -> gather reproduces the unsharded result
bit-for-bit, including uneven splits (units not divisible by the world size)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_pldi_tangzwjzyz22_b200.dist import shard_bounds


def test_shard_bounds_partition():
    for units in (1, 2, 3, 7, 8, 64):
        for world in (1, 2, 3, 4, 8):
            spans = [shard_bounds(units, world, r) for r in range(world)]
            assert spans[0][0] == 0 and spans[-1][1] == units
            for (a, b), (c, _) in zip(spans, spans[1:]):
                assert b == c and b >= a
            sizes = [b - a for a, b in spans]
            assert max(sizes) - min(sizes) <= 1


def _oracle_compute(q, k, v, g, w, dil):
    import oracle
    o, l_ = oracle.fwd(q.numpy(), k.numpy(), v.numpy(), w, dil)
    dq, dk, dv = oracle.bwd(q.numpy(), k.numpy(), v.numpy(), o, l_, g.numpy(), w, dil)
    return tuple(torch.from_numpy(x) for x in (o, l_, dq, dk, dv))


def _worker(rank, world, port, B, H, L, d, w, dil, result_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_pldi_tangzwjzyz22_b200.dist import sharded_fwd_bwd
        from synth import WinAttnShape, make_inputs
        x = make_inputs(WinAttnShape(B, H, L, d, w, dil), 3, "f32")
        args = [torch.from_numpy(x[n]) for n in ("q64", "k64", "v64", "dout64")] if rank == 0 \
            else [None] * 4
        res = sharded_fwd_bwd(*args, w, dil, shape=(B, H, L, d), dtype=torch.float64,
                              device=torch.device("cpu"), compute=_oracle_compute)
        if rank == 0:
            full = _oracle_compute(*(torch.from_numpy(x[n]) for n in ("q64", "k64", "v64", "dout64")),
                                   w, dil)
            ok = all(torch.equal(a, b) for a, b in zip(res, full))
            result_q.put(ok)
    finally:
        dist.destroy_process_group()


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.parametrize("B,H", [(1, 2), (1, 3), (2, 3)])
def test_sharded_fwd_bwd_gloo_world2(B, H):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, B, H, 40, 8, 3, 2, q)) for r in range(2)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert q.get(timeout=5) is True


# ---------------------------------------------------------------- context (sequence) parallel
def _oracle_fwd_t(q, k, v, w, dil):
    import oracle
    o, l_ = oracle.fwd(q.numpy(), k.numpy(), v.numpy(), w, dil)
    return torch.from_numpy(o), torch.from_numpy(l_)


def _oracle_bwd_t(q, k, v, o, l_, g, w, dil):
    import oracle
    r = oracle.bwd(q.numpy(), k.numpy(), v.numpy(), o.numpy(), l_.numpy(), g.numpy(), w, dil)
    return tuple(torch.from_numpy(x) for x in r)


def _cp_worker(rank, world, port, B, H, L, d, w, dil, result_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_pldi_tangzwjzyz22_b200.dist import cp_bwd, cp_fwd, seq_bounds
        from synth import WinAttnShape, make_inputs
        x = make_inputs(WinAttnShape(B, H, L, d, w, dil), 5, "f32")
        full = {n: torch.from_numpy(x[n + "64"]) for n in ("q", "k", "v", "dout")}
        lo, hi = seq_bounds(L, world, rank)
        loc = {n: t[:, :, lo:hi].contiguous() for n, t in full.items()}
        out, lse = cp_fwd(loc["q"], loc["k"], loc["v"], w, dil, L, fwd_fn=_oracle_fwd_t)
        dq, dk, dv = cp_bwd(loc["q"], loc["k"], loc["v"], out, lse, loc["dout"], w, dil, L,
                            bwd_fn=_oracle_bwd_t)
        ro, rl = _oracle_fwd_t(full["q"], full["k"], full["v"], w, dil)
        rdq, rdk, rdv = _oracle_bwd_t(full["q"], full["k"], full["v"], ro, rl, full["dout"], w, dil)
        errs = [float((a - b[..., lo:hi] if a.dim() == 3 else a - b[:, :, lo:hi]).abs().max())
                for a, b in ((out, ro), (lse, rl), (dq, rdq), (dk, rdk), (dv, rdv))]
        result_q.put((rank, errs))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,shape", [
    (2, (1, 2, 200, 16, 8, 1)),
    (3, (2, 1, 301, 8, 5, 3)),      # dilation: halo of w * dilation rows, uneven slices
    (4, (1, 1, 260, 16, 16, 2)),
])
def test_context_parallel_matches_full_sequence(world, shape):
    """Sequence-sharded fwd + bwd with one halo exchange per direction (dist.cp_fwd / cp_bwd),
    the per-rank compute being the fp64 oracle: every rank's rows of out, lse, dq, dk, dv equal
    the unsharded oracle's up to fp64 summation order."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_cp_worker, args=(r, world, port, *shape, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, errs in res:
        assert max(errs) < 1e-12, (rank, errs)


def _halo_check_worker(rank, world, port, L, w, dil, result_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_pldi_tangzwjzyz22_b200.dist import cp_fwd, seq_bounds
        lo, hi = seq_bounds(L, world, rank)
        x = torch.zeros(1, 1, hi - lo, 8, dtype=torch.float64)
        try:
            cp_fwd(x, x, x, w, dil, L, fwd_fn=_oracle_fwd_t)
            result_q.put((rank, "ran"))
        except ValueError:
            result_q.put((rank, "raised"))
    finally:
        dist.destroy_process_group()


def test_context_parallel_rejects_short_slices_on_every_rank():
    """L = 11 over 3 ranks (slices 4 / 4 / 3) with a halo of 4 rows: the smallest slice cannot
    hold a halo, and EVERY rank must raise before any communication (a rank-dependent check
    would leave the others waiting on it)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_halo_check_worker, args=(r, 3, port, 11, 4, 1, q)) for r in range(3)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=120) for _ in range(3))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert res == {0: "raised", 1: "raised", 2: "raised"}
