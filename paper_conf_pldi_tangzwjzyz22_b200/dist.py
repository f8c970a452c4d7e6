"""Multi-GPU sharding of window attention by (batch, head) unit.

Units u = b*H + h are independent: Fig. 8 has no term that crosses
heads or batches.  So the data-parallel job needs no collective on its compute path; this
module provides the north_star's end-to-end variant where rank 0 owns the full tensors:

    scatter q, k, v, dout (contiguous unit slabs of [B*H, L, d]) from rank 0
    -> each rank: one ft_winattn_fwd + one ft_winattn_bwd on its slab
    -> gather out, lse, dq, dk, dv back to rank 0

Slabs are contiguous in the [B, H, L, d] layout, so no packing copies are made except the
zero padding that makes the last slab as long as the others (NCCL scatter/gather need
equal-size buffers).  Works with any torch.distributed backend (nccl on GPUs, gloo in the
CPU tests).
"""
from __future__ import annotations

from typing import Callable, Sequence

import torch
import torch.distributed as dist


def shard_bounds(units: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous block [lo, hi) of units owned by `rank` (balanced to within one unit)."""
    base, extra = divmod(units, world)
    lo = rank * base + min(rank, extra)
    hi = lo + base + (1 if rank < extra else 0)
    return lo, hi


def _slab_len(units: int, world: int) -> int:
    return -(-units // world)


def scatter_units(full: torch.Tensor | None, units: int, tail_shape: Sequence[int],
                  dtype: torch.dtype, device, src: int = 0) -> torch.Tensor:
    """Scatter a [units, *tail] tensor held by `src` into per-rank unit slabs."""
    world, rank = dist.get_world_size(), dist.get_rank()
    n = _slab_len(units, world)
    recv = torch.empty((n, *tail_shape), dtype=dtype, device=device)
    chunks = None
    if rank == src:
        flat = full.reshape(units, *tail_shape)
        chunks = []
        for r in range(world):
            lo, hi = shard_bounds(units, world, r)
            c = torch.zeros((n, *tail_shape), dtype=dtype, device=device)
            c[: hi - lo].copy_(flat[lo:hi])
            chunks.append(c)
    dist.scatter(recv, chunks, src=src)
    lo, hi = shard_bounds(units, world, rank)
    return recv[: hi - lo]


def gather_units(local: torch.Tensor, units: int, dst: int = 0) -> torch.Tensor | None:
    """Gather per-rank unit slabs back into a [units, *tail] tensor on `dst`."""
    world, rank = dist.get_world_size(), dist.get_rank()
    n = _slab_len(units, world)
    send = torch.zeros((n, *local.shape[1:]), dtype=local.dtype, device=local.device)
    send[: local.shape[0]].copy_(local)
    bufs = None
    if rank == dst:
        bufs = [torch.empty_like(send) for _ in range(world)]
    dist.gather(send, bufs, dst=dst)
    if rank != dst:
        return None
    parts = []
    for r in range(world):
        lo, hi = shard_bounds(units, world, r)
        parts.append(bufs[r][: hi - lo])
    return torch.cat(parts, dim=0)


def _default_compute(q, k, v, g, w, dilation):
    from . import bwd, fwd
    out, lse = fwd(q, k, v, w, dilation)
    dq, dk, dv = bwd(q, k, v, out, lse, g, w, dilation)
    return out, lse, dq, dk, dv


def sharded_fwd_bwd(q, k, v, dout, w: int, dilation: int = 1, shape=None, dtype=None,
                    device=None, src: int = 0,
                    compute: Callable | None = None):
    """End-to-end sharded fwd+bwd.  On `src`, q/k/v/dout are the full [B,H,L,d] tensors
    (other ranks pass None together with shape/dtype).  Returns (out, lse, dq, dk, dv) on
    `src` and None elsewhere.  `compute(q,k,v,g,w,dil)` runs on each [1, n, L, d] slab."""
    rank = dist.get_rank()
    if rank == src:
        shape, dtype, device = tuple(q.shape), q.dtype, q.device
    B, H, L, d = shape
    units = B * H
    compute = compute or _default_compute
    slabs = [scatter_units(x if rank == src else None, units, (L, d), dtype, device, src)
             for x in (q, k, v, dout)]
    n = slabs[0].shape[0]
    if n > 0:
        res = compute(*(s.reshape(1, n, L, d).contiguous() for s in slabs), w, dilation)
        out, lse, dq, dk, dv = (r.reshape(n, *r.shape[2:]) for r in res)
    else:
        out, dq, dk, dv = (torch.empty((0, L, d), dtype=dtype, device=device) for _ in range(4))
        lse = torch.empty((0, L), dtype=torch.float32, device=device)
    got = [gather_units(t, units, src) for t in (out, lse, dq, dk, dv)]
    if rank != src:
        return None
    o, l_, a, b, c = got
    return (o.reshape(B, H, L, d), l_.reshape(B, H, L), a.reshape(B, H, L, d),
            b.reshape(B, H, L, d), c.reshape(B, H, L, d))
