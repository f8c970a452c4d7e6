"""SubdivNet's circular difference on B200 -- Python binding of include/ft_subdiv.h.

Argument marshalling only: the forward and backward run in the library's CUDA kernels
(csrc/subdiv.cu); there is no CPU or PyTorch fallback.

    y[i, k] = sum_j |e[adj[i, j], k] - e[adj[i, (j+1) % 3], k]|      (Fig. 2)
"""
from __future__ import annotations

import ctypes

import torch

from . import FT_BF16, FT_F32, FtError, _check, _stream, load_library

__all__ = ["circdiff_fwd", "circdiff_bwd", "CircDiff", "circdiff"]


def _lib():
    lib = load_library()
    if not getattr(lib, "_subdiv_sigs", False):
        vp, i64 = ctypes.c_void_p, ctypes.c_int64
        lib.ft_subdiv_circdiff_fwd.argtypes = [vp, vp, vp, i64, i64, ctypes.c_int, vp]
        lib.ft_subdiv_circdiff_fwd.restype = ctypes.c_int
        lib.ft_subdiv_circdiff_bwd.argtypes = [vp] * 4 + [i64, i64, ctypes.c_int, ctypes.c_int, vp,
                                                          ctypes.c_size_t, vp]
        lib.ft_subdiv_circdiff_bwd.restype = ctypes.c_int
        lib.ft_subdiv_circdiff_bwd_workspace_bytes.argtypes = [i64, i64, ctypes.c_int]
        lib.ft_subdiv_circdiff_bwd_workspace_bytes.restype = ctypes.c_size_t
        lib._subdiv_sigs = True
    return lib


def _code(t: torch.Tensor) -> int:
    if t.dtype == torch.float32:
        return FT_F32
    if t.dtype == torch.bfloat16:
        return FT_BF16
    raise TypeError(f"unsupported dtype {t.dtype}")


def _check_args(e: torch.Tensor, adj: torch.Tensor):
    if not (e.is_cuda and adj.is_cuda and e.device == adj.device):
        raise ValueError("e and adj must be CUDA tensors on one device")
    if e.dim() != 2 or adj.shape != (e.shape[0], 3) or adj.dtype != torch.int32:
        raise ValueError("expected e [n_faces, n_feats] and adj int32 [n_faces, 3]")
    if not (e.is_contiguous() and adj.is_contiguous()):
        raise ValueError("tensors must be contiguous")


def circdiff_fwd(e: torch.Tensor, adj: torch.Tensor, y: torch.Tensor | None = None) -> torch.Tensor:
    _check_args(e, adj)
    y = torch.empty_like(e) if y is None else y
    n, f = e.shape
    _check(_lib().ft_subdiv_circdiff_fwd(e.data_ptr(), adj.data_ptr(), y.data_ptr(), n, f, _code(e),
                                         _stream(e.device)))
    return y


def circdiff_bwd(e: torch.Tensor, adj: torch.Tensor, dy: torch.Tensor, de: torch.Tensor | None = None,
                 workspace: torch.Tensor | None = None, symmetric: bool = False) -> torch.Tensor:
    """de for the loss sum(y * dy).  symmetric=True: adj is a closed manifold mesh's edge
    adjacency (gather kernel, deterministic); False: any adjacency (atomic scatter)."""
    _check_args(e, adj)
    if dy.shape != e.shape or dy.dtype != e.dtype or not dy.is_contiguous():
        raise ValueError("dy must match e")
    de = torch.empty_like(e) if de is None else de
    n, f = e.shape
    lib = _lib()
    need = int(lib.ft_subdiv_circdiff_bwd_workspace_bytes(n, f, _code(e)))
    if need and (workspace is None or workspace.numel() * workspace.element_size() < need):
        workspace = torch.empty(need, dtype=torch.uint8, device=e.device)
    wp = workspace.data_ptr() if need else None
    wb = workspace.numel() * workspace.element_size() if need else 0
    _check(lib.ft_subdiv_circdiff_bwd(e.data_ptr(), adj.data_ptr(), dy.data_ptr(), de.data_ptr(), n, f,
                                      _code(e), int(symmetric), wp, wb, _stream(e.device)))
    return de


class CircDiff(torch.autograd.Function):
    @staticmethod
    def forward(ctx, e, adj, symmetric: bool = False):
        e = e.contiguous()
        ctx.save_for_backward(e, adj)
        ctx.symmetric = symmetric
        return circdiff_fwd(e, adj)

    @staticmethod
    def backward(ctx, dy):
        e, adj = ctx.saved_tensors
        return circdiff_bwd(e, adj, dy.contiguous(), symmetric=ctx.symmetric), None, None


def circdiff(e, adj, symmetric: bool = False):
    return CircDiff.apply(e, adj, symmetric)
