"""Multi-process host logic of dist.py with the CUDA kernels as the per-rank compute (-m gpu).

gpurun provides one GPU, so both ranks run on cuda:0 and exchange over gloo (CPU tensors):
each rank's compute moves its slab to the GPU, runs ft_winattn through the C ABI and brings the
result back.  (batch, head) sharding must reproduce the one-call result bit for bit (every unit
is computed by the same kernels on the same data); context parallelism (sequence slices with one
halo exchange per direction, dK / dV of the halo rows returned to their owners) must match the
fp64 oracle within the bf16 / fp32 tolerances of tests/_util.py."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _gpu_fns(dtype):
    """fp32 CPU tensors in and out; the kernels run on cuda:0 in `dtype` (bf16 values are exact in fp32)"""
    import paper_conf_pldi_tangzwjzyz22_b200 as ft
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    dev = torch.device("cuda:0")

    def up(t):
        return t.to(dev).to(tdt).contiguous()

    def down(t):
        return t.float().cpu()

    def fwd_fn(q, k, v, w, dil):
        o, l_ = ft.fwd(up(q), up(k), up(v), w, dil)
        return down(o), l_.cpu()

    def bwd_fn(q, k, v, o, l_, g, w, dil):
        r = ft.bwd(up(q), up(k), up(v), up(o), l_.to(dev).contiguous(), up(g), w, dil)
        return tuple(down(x) for x in r)

    def compute(q, k, v, g, w, dil):
        o, l_ = fwd_fn(q, k, v, w, dil)
        return (o, l_) + bwd_fn(q, k, v, o, l_, g, w, dil)

    return fwd_fn, bwd_fn, compute


def _inputs(shape, dtype, seed):
    from synth import WinAttnShape, make_inputs
    x = make_inputs(WinAttnShape(*shape), seed, dtype)
    return {n: x[n].float() for n in ("q", "k", "v", "dout")}, x


def _shard_worker(rank, world, port, shape, dtype, result_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_pldi_tangzwjzyz22_b200.dist import sharded_fwd_bwd
        _, _, compute = _gpu_fns(dtype)
        t, _ = _inputs(shape, dtype, 51)
        B, H, L, d, w, dil = shape
        args = [t[n] for n in ("q", "k", "v", "dout")] if rank == 0 else [None] * 4
        res = sharded_fwd_bwd(*args, w, dil, shape=(B, H, L, d), dtype=torch.float32,
                              device=torch.device("cpu"), compute=compute)
        if rank == 0:
            full = compute(*(t[n] for n in ("q", "k", "v", "dout")), w, dil)
            result_q.put(all(torch.equal(a, b) for a, b in zip(res, full)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("shape,dtype", [((1, 3, 700, 512, 32, 1), "bf16"), ((2, 3, 900, 64, 32, 2), "bf16"),
                                         ((1, 4, 600, 64, 100, 1), "bf16"), ((1, 3, 300, 64, 16, 1), "f32"),
                                         ((1, 2, 700, 512, 32, 1), "f32")],   # fp32 tensor cores + dS tape
                         ids=lambda s: "x".join(map(str, s)) if isinstance(s, tuple) else s)
def test_sharded_fwd_bwd_cuda_world2(shape, dtype):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_shard_worker, args=(r, 2, port, shape, dtype, q)) for r in range(2)]
    for p in procs:
        p.start()
    ok = q.get(timeout=300)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert ok is True


def _cp_worker(rank, world, port, shape, dtype, result_q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from _util import compare
        from paper_conf_pldi_tangzwjzyz22_b200.dist import cp_bwd, cp_fwd, seq_bounds
        fwd_fn, bwd_fn, _ = _gpu_fns(dtype)
        t, x = _inputs(shape, dtype, 52)
        B, H, L, d, w, dil = shape
        lo, hi = seq_bounds(L, world, rank)
        loc = {n: v[:, :, lo:hi].contiguous() for n, v in t.items()}
        out, lse = cp_fwd(loc["q"], loc["k"], loc["v"], w, dil, L, fwd_fn=fwd_fn)
        dq, dk, dv = cp_bwd(loc["q"], loc["k"], loc["v"], out, lse, loc["dout"], w, dil, L, bwd_fn=bwd_fn)
        ro, rl = oracle.fwd(x["q64"], x["k64"], x["v64"], w, dil)
        rq, rk, rv = oracle.bwd(x["q64"], x["k64"], x["v64"], ro, rl, x["dout64"], w, dil)
        msg = "ok"
        try:
            for n, a, r in (("out", out, ro), ("lse", lse, rl), ("dq", dq, rq), ("dk", dk, rk), ("dv", dv, rv)):
                compare(n, a.double().numpy(), r[:, :, lo:hi], dtype)
        except AssertionError as ex:
            msg = str(ex)[:400]
        result_q.put((rank, msg))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,shape,dtype", [(2, (1, 2, 1000, 512, 32, 1), "bf16"),
                                               (3, (2, 2, 1500, 64, 32, 3), "bf16"),
                                               (2, (1, 2, 1200, 64, 100, 1), "bf16"),
                                               (2, (1, 2, 500, 64, 16, 2), "f32"),
                                               (2, (1, 2, 800, 256, 32, 1), "f32"),    # fp32 tensor cores + dS tape
                                               (2, (1, 2, 1400, 64, 150, 1), "f32"),   # fp32 WIDE steps
                                               (2, (1, 1, 1000, 128, 100, 1), "bf16")],  # d = 128 wide kernels
                         ids=lambda s: "x".join(map(str, s)) if isinstance(s, tuple) else str(s))
def test_context_parallel_cuda(world, shape, dtype):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_cp_worker, args=(r, world, port, shape, dtype, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
    for rank, msg in res:
        assert msg == "ok", (rank, msg)
