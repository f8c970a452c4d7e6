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


# ------------------------------------------------------------------ sequence (context) parallel
# when B*H is smaller than the number of GPUs, or L is very long, each
# rank holds a contiguous slice of the SEQUENCE of every (batch, head) unit instead.  A query
# row attends only to keys within h = w * dilation rows (reading A1/A4), so a rank
# needs h halo rows of K and V from each neighbour -- one NCCL point-to-point exchange -- and,
# in the backward, returns the dK / dV its queries produced for the neighbours' rows.
#
# The local call runs the ordinary single-GPU kernels on the extended slice [halo | own | halo]:
#   forward : q halo rows are zero; their outputs are discarded.
#   backward: q, out, dout of the halo rows are zero and their lse is 0, so P = 1 on their band
#             but dP = dout . v = 0 and D = 0, hence dS = 0 and P^T dout = 0 -- halo queries add
#             nothing to dK / dV, which therefore hold exactly the contributions of this rank's
#             queries; the halo rows' dK / dV go back to their owners and are added there.


def seq_bounds(L: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous rows [lo, hi) of the sequence owned by `rank` (balanced to within one row)."""
    return shard_bounds(L, world, rank)


def _neighbour_exchange(send_left: torch.Tensor | None, send_right: torch.Tensor | None,
                        recv_left_shape, recv_right_shape, group=None):
    """Send `send_left` to rank-1 and `send_right` to rank+1; receive tensors of the given shapes
    (None = no neighbour) from rank-1 and rank+1.  One batched set of P2P ops (NCCL send/recv
    over NVLink on GPUs, gloo on CPU)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    ops, rl, rr = [], None, None
    ref = send_left if send_left is not None else send_right
    if recv_left_shape is not None:
        rl = torch.empty(recv_left_shape, dtype=ref.dtype, device=ref.device)
        ops.append(dist.P2POp(dist.irecv, rl, rank - 1, group))
    if recv_right_shape is not None:
        rr = torch.empty(recv_right_shape, dtype=ref.dtype, device=ref.device)
        ops.append(dist.P2POp(dist.irecv, rr, rank + 1, group))
    if send_left is not None and rank > 0:
        ops.append(dist.P2POp(dist.isend, send_left.contiguous(), rank - 1, group))
    if send_right is not None and rank < world - 1:
        ops.append(dist.P2POp(dist.isend, send_right.contiguous(), rank + 1, group))
    if ops:
        for r in dist.batch_isend_irecv(ops):
            r.wait()
    return rl, rr


def _halos(L: int, w: int, dilation: int, group=None):
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    lo, hi = seq_bounds(L, world, rank)
    h = min(w * dilation, L)
    hl = min(h, lo)              # rows of rank-1 this rank needs
    hr = min(h, L - hi)          # rows of rank+1
    # rank-independent condition (the smallest slice, L // world rows, must hold a whole halo),
    # so that every rank raises before any communication instead of some ranks waiting on a
    # peer that raised
    if world > 1 and L // world < h:
        raise ValueError(f"context parallel needs every rank to own >= w*dilation = {h} rows "
                         f"(L = {L} over {world} ranks gives {L // world})")
    return lo, hi, hl, hr


def _extend(x: torch.Tensor, hl: int, hr: int, group=None, zero_halo: bool = False):
    """[B, H, n, ...] local slice -> [B, H, hl + n + hr, ...] with the neighbours' rows (or zeros)."""
    B, H, n = x.shape[:3]
    tail = tuple(x.shape[3:])
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    if zero_halo:
        left = x.new_zeros((B, H, hl) + tail)
        right = x.new_zeros((B, H, hr) + tail)
    else:
        # my first rows are rank-1's right halo and my last rows rank+1's left halo; _halos
        # guarantees every rank owns >= h rows, so both sides of each link agree on the size
        send_l = x[:, :, :hl] if rank > 0 else None
        send_r = x[:, :, n - hr:] if rank < world - 1 else None
        left, right = _neighbour_exchange(send_l, send_r,
                                          (B, H, hl) + tail if hl > 0 else None,
                                          (B, H, hr) + tail if hr > 0 else None, group)
        left = left if left is not None else x.new_zeros((B, H, 0) + tail)
        right = right if right is not None else x.new_zeros((B, H, 0) + tail)
    return torch.cat([left, x, right], dim=2).contiguous()


def cp_fwd(q, k, v, w: int, dilation: int, L: int, fwd_fn: Callable | None = None, group=None):
    """Context-parallel forward.  q, k, v: this rank's rows [lo, hi) of the [B, H, L, d] tensors
    (seq_bounds).  Returns (out, lse) for those rows.  `fwd_fn(q, k, v, w, dil)` is the local
    single-device forward (default: the CUDA library)."""
    if fwd_fn is None:
        from . import fwd as fwd_fn
    lo, hi, hl, hr = _halos(L, w, dilation, group)
    n = hi - lo
    ke, ve = _extend(k, hl, hr, group), _extend(v, hl, hr, group)
    qe = _extend(q, hl, hr, group, zero_halo=True)
    out, lse = fwd_fn(qe, ke, ve, w, dilation)
    return out[:, :, hl:hl + n].contiguous(), lse[:, :, hl:hl + n].contiguous()


def cp_bwd(q, k, v, out, lse, dout, w: int, dilation: int, L: int, bwd_fn: Callable | None = None,
           group=None):
    """Context-parallel backward over this rank's rows; returns (dq, dk, dv) for them.  dK / dV
    of the halo rows (this rank's queries' contributions to its neighbours' keys) are sent back
    and added by their owners."""
    if bwd_fn is None:
        from . import bwd as bwd_fn
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    lo, hi, hl, hr = _halos(L, w, dilation, group)
    n = hi - lo
    ke, ve = _extend(k, hl, hr, group), _extend(v, hl, hr, group)
    qe, oe, ge = (_extend(t, hl, hr, group, zero_halo=True) for t in (q, out, dout))
    le = _extend(lse, hl, hr, group, zero_halo=True)
    dqe, dke, dve = bwd_fn(qe, ke, ve, oe, le, ge, w, dilation)
    dq = dqe[:, :, hl:hl + n].contiguous()
    dk = dke[:, :, hl:hl + n].clone()
    dv = dve[:, :, hl:hl + n].clone()
    # halo parts back to their owners: my left halo rows are rank-1's last rows, the right
    # halo rows rank+1's first rows
    hkv_l = torch.cat([dke[:, :, :hl], dve[:, :, :hl]], dim=-1) if rank > 0 else None
    hkv_r = torch.cat([dke[:, :, hl + n:], dve[:, :, hl + n:]], dim=-1) if rank < world - 1 else None
    need_prev = hl      # my first rows = rank-1's right halo (same size, see _halos)
    need_next = hr      # my last rows = rank+1's left halo
    d2 = dk.shape[-1] * 2
    B, H = dk.shape[:2]
    from_prev, from_next = _neighbour_exchange(
        hkv_l, hkv_r,
        (B, H, need_prev, d2) if need_prev > 0 else None,
        (B, H, need_next, d2) if need_next > 0 else None, group)
    d = dk.shape[-1]
    if from_prev is not None:   # rank-1's queries -> my first rows
        dk[:, :, :need_prev] += from_prev[..., :d].to(dk.dtype)
        dv[:, :, :need_prev] += from_prev[..., d:].to(dv.dtype)
    if from_next is not None:   # rank+1's queries -> my last rows
        dk[:, :, n - need_next:] += from_next[..., :d].to(dk.dtype)
        dv[:, :, n - need_next:] += from_next[..., d:].to(dv.dtype)
    return dq, dk, dv
