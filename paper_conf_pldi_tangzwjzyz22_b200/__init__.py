"""B200-native banded (dilated) sliding-window attention — Python binding of ft_winattn.

The compute lives in ``libft_winattn.so`` (hand-written sm_100a CUDA kernels behind the
C ABI of ``include/ft_winattn.h``).  This module only marshals arguments: it checks
dtype / device / contiguity, allocates outputs with PyTorch and calls the C entry points
through ctypes on ``torch.cuda.current_stream()``.  There is no CPU or PyTorch fallback:
if the library is missing or a call fails, it raises.

Operation (Fig. 5/8, lines 167-231): for each (batch, head) and
query row i, attend to keys j = i + k*dilation with |k| <= w and 0 <= j < L, unscaled
logits q_i.k_j, row softmax with saved log-sum-exp, weighted sum over V; the backward
recomputes P from lse and returns dq, dk, dv.
"""
from __future__ import annotations

import ctypes
import os

import torch

__all__ = ["fwd", "bwd", "fwd_bwd", "knobs", "debug_set", "debug_get", "fwd_tape", "bwd_tape", "tape_bytes", "plan", "profile_events", "WinAttn", "win_attn", "lib_path", "load_library",
           "FT_F32", "FT_BF16", "PATH_SIMT", "PATH_TC", "FtError"]

_PKG = os.path.dirname(os.path.abspath(__file__))
_LIB_NAME = "libft_winattn.so"

FT_F32, FT_BF16 = 0, 1
PATH_SIMT, PATH_TC = 0, 1
_STATUS = {0: "FT_OK", 1: "FT_ERR_INVALID_VALUE", 2: "FT_ERR_NOT_SUPPORTED",
           3: "FT_ERR_MISALIGNED", 4: "FT_ERR_CUDA"}

_lib = None


class FtError(RuntimeError):
    def __init__(self, status: int, msg: str):
        super().__init__(msg)
        self.status = status


def lib_path() -> str:
    """The in-tree library; FT_WINATTN_LIB names another build of it (A/B timing aid)."""
    return os.environ.get("FT_WINATTN_LIB") or os.path.join(_PKG, _LIB_NAME)


def load_library(build_if_missing: bool = False):
    """Load (optionally build) the in-tree shared library and declare its C signatures."""
    global _lib
    if _lib is not None:
        return _lib
    path = lib_path()
    if not os.path.exists(path):
        if not build_if_missing:
            raise RuntimeError(f"{path} is missing: build it with "
                               "`python -m paper_conf_pldi_tangzwjzyz22_b200.build`")
        from . import build as _build
        _build.build()
    lib = ctypes.CDLL(path)
    i64, vp, sz = ctypes.c_int64, ctypes.c_void_p, ctypes.c_size_t
    fp = ctypes.c_void_p
    lib.ft_winattn_fwd.argtypes = [vp, vp, vp, vp, fp] + [i64] * 6 + [ctypes.c_int, vp]
    lib.ft_winattn_fwd.restype = ctypes.c_int
    lib.ft_winattn_bwd.argtypes = [vp] * 9 + [i64] * 6 + [ctypes.c_int, vp, sz, vp]
    lib.ft_winattn_bwd.restype = ctypes.c_int
    lib.ft_winattn_fwd_bwd.argtypes = [vp] * 9 + [i64] * 6 + [ctypes.c_int, vp, sz, vp]
    lib.ft_winattn_fwd_bwd.restype = ctypes.c_int
    lib.ft_winattn_debug_set.argtypes = [ctypes.c_int, ctypes.c_int]
    lib.ft_winattn_debug_set.restype = ctypes.c_int
    lib.ft_winattn_debug_get.argtypes = [ctypes.c_int]
    lib.ft_winattn_debug_get.restype = ctypes.c_int
    lib.ft_winattn_fwd_mixed.argtypes = [vp, vp, vp, vp, fp] + [i64] * 7 + [ctypes.c_int, vp]
    lib.ft_winattn_fwd_mixed.restype = ctypes.c_int
    lib.ft_winattn_bwd_mixed.argtypes = [vp] * 9 + [i64] * 7 + [ctypes.c_int, vp, sz, vp]
    lib.ft_winattn_bwd_mixed.restype = ctypes.c_int
    lib.ft_winattn_tape_bytes.argtypes = [i64] * 4
    lib.ft_winattn_tape_bytes.restype = sz
    lib.ft_winattn_fwd_tape.argtypes = [vp, vp, vp, vp, fp, fp] + [i64] * 6 + [ctypes.c_int, vp]
    lib.ft_winattn_fwd_tape.restype = ctypes.c_int
    lib.ft_winattn_bwd_tape.argtypes = [vp] * 10 + [i64] * 6 + [ctypes.c_int, vp, sz, vp]
    lib.ft_winattn_bwd_tape.restype = ctypes.c_int
    lib.ft_winattn_bwd_workspace_bytes.argtypes = [i64] * 6 + [ctypes.c_int]
    lib.ft_winattn_bwd_workspace_bytes.restype = sz
    lib.ft_winattn_plan.argtypes = [ctypes.c_int] + [i64] * 6 + [ctypes.c_int,
                                                                 ctypes.POINTER(ctypes.c_int),
                                                                 ctypes.POINTER(ctypes.c_int)]
    lib.ft_winattn_plan.restype = ctypes.c_int
    lib.ft_status_str.argtypes = [ctypes.c_int]
    lib.ft_status_str.restype = ctypes.c_char_p
    lib.ft_winattn_abi_version.restype = ctypes.c_int
    lib.ft_winattn_profile_events.argtypes = [ctypes.c_void_p, ctypes.c_int]
    lib.ft_winattn_profile_events.restype = ctypes.c_int
    _lib = lib
    return lib


_KNOBS = {"path": 0, "pdl": 1, "narrow": 2, "wide": 3, "side": 4, "dstape": 5}
_PATHS = {"auto": 0, "simt": 1, "tc": 2}


def debug_set(name: str, value) -> None:
    """Set a debug / A-B knob of include/ft_winattn.h (path: auto|simt|tc; pdl, narrow, wide,
    side: 0|1).  Process-wide; every setting computes the same result."""
    v = _PATHS[value] if name == "path" and isinstance(value, str) else int(value)
    _check(load_library().ft_winattn_debug_set(_KNOBS[name], v))


def debug_get(name: str) -> int:
    return int(load_library().ft_winattn_debug_get(_KNOBS[name]))


class knobs:
    """Context manager: ``with knobs(path="simt", pdl=0): ...`` sets debug knobs and restores
    the previous values on exit."""

    def __init__(self, **kv):
        self.kv = kv

    def __enter__(self):
        self.old = {k: debug_get(k) for k in self.kv}
        for k, v in self.kv.items():
            debug_set(k, v)
        return self

    def __exit__(self, *a):
        for k, v in self.old.items():
            debug_set(k, v)


def _dtype_code(t: torch.Tensor) -> int:
    if t.dtype == torch.float32:
        return FT_F32
    if t.dtype == torch.bfloat16:
        return FT_BF16
    raise TypeError(f"unsupported dtype {t.dtype} (expected float32 or bfloat16)")


def _check(status: int):
    if status != 0:
        msg = load_library().ft_status_str(status).decode()
        raise FtError(status, msg)


def _check_inputs(*ts: torch.Tensor):
    ref = ts[0]
    if ref.dim() != 4:
        raise ValueError("expected [batch, heads, seq_len, d] tensors")
    for t in ts:
        if not t.is_cuda:
            raise ValueError("ft_winattn tensors must be CUDA tensors")
        if t.shape != ref.shape or t.dtype != ref.dtype or t.device != ref.device:
            raise ValueError("q, k, v (and out, dout) must share shape, dtype and device")
        if not t.is_contiguous():
            raise ValueError("ft_winattn tensors must be contiguous")


def _stream(device) -> int:
    return torch.cuda.current_stream(device).cuda_stream


class profile_events:
    """Context manager: record ``events[i]`` (torch.cuda.Event, timing enabled) right after
    the i-th kernel launch of every fwd/bwd call made inside the block (C ABI
    ft_winattn_profile_events).  Use a fresh list per call to time each launch."""

    def __init__(self, events):
        self.events = list(events)
        for e in self.events:
            if not e.cuda_event:
                e.record()   # torch creates the CUDA event lazily; materialise its handle
        self._arr = (ctypes.c_void_p * max(1, len(self.events)))(
            *[ctypes.c_void_p(e.cuda_event) for e in self.events])

    def __enter__(self):
        load_library().ft_winattn_profile_events(ctypes.cast(self._arr, ctypes.c_void_p),
                                                 len(self.events))
        return self

    def __exit__(self, *a):
        load_library().ft_winattn_profile_events(None, 0)


def plan(is_bwd: bool, batch: int, heads: int, seq_len: int, d: int, w: int, dilation: int,
         dtype) -> tuple[int, int]:
    """(path, number of kernel launches) a call with these arguments would make."""
    code = dtype if isinstance(dtype, int) else (FT_F32 if dtype == torch.float32 else FT_BF16)
    path, n = ctypes.c_int(0), ctypes.c_int(0)
    _check(load_library().ft_winattn_plan(int(is_bwd), batch, heads, seq_len, d, w, dilation,
                                          code, ctypes.byref(path), ctypes.byref(n)))
    return path.value, n.value


def fwd(q: torch.Tensor, k: torch.Tensor, v: torch.Tensor, w: int, dilation: int = 1,
        out: torch.Tensor | None = None, lse: torch.Tensor | None = None,
        dilated_heads: int | None = None):
    """Forward: returns (out [B,H,L,d] in q.dtype, lse [B,H,L] fp32).  With ``dilated_heads``
    only heads [0, dilated_heads) use ``dilation`` and the rest dilation 1
    (ft_winattn_fwd_mixed)."""
    _check_inputs(q, k, v)
    B, H, L, d = q.shape
    if out is None:
        out = torch.empty_like(q)
    if lse is None:
        lse = torch.empty((B, H, L), dtype=torch.float32, device=q.device)
    lib = load_library()
    if dilated_heads is None:
        _check(lib.ft_winattn_fwd(q.data_ptr(), k.data_ptr(), v.data_ptr(), out.data_ptr(),
                                  lse.data_ptr(), B, H, L, d, int(w), int(dilation),
                                  _dtype_code(q), _stream(q.device)))
    else:
        _check(lib.ft_winattn_fwd_mixed(q.data_ptr(), k.data_ptr(), v.data_ptr(), out.data_ptr(),
                                        lse.data_ptr(), B, H, L, d, int(w), int(dilation),
                                        int(dilated_heads), _dtype_code(q), _stream(q.device)))
    return out, lse


def workspace_bytes(q: torch.Tensor, w: int, dilation: int = 1) -> int:
    B, H, L, d = q.shape
    return int(load_library().ft_winattn_bwd_workspace_bytes(B, H, L, d, int(w), int(dilation),
                                                             _dtype_code(q)))


def bwd(q, k, v, out, lse, dout, w: int, dilation: int = 1, dq=None, dk=None, dv=None,
        workspace: torch.Tensor | None = None, dilated_heads: int | None = None):
    """Backward: returns (dq, dk, dv) in q.dtype (``dilated_heads``: see fwd)."""
    _check_inputs(q, k, v, out, dout)
    B, H, L, d = q.shape
    if lse.dtype != torch.float32 or not lse.is_contiguous() or lse.shape != (B, H, L):
        raise ValueError("lse must be a contiguous fp32 [B, H, L] tensor")
    dq = torch.empty_like(q) if dq is None else dq
    dk = torch.empty_like(q) if dk is None else dk
    dv = torch.empty_like(q) if dv is None else dv
    wsb = workspace_bytes(q, w, dilation)
    if workspace is None or workspace.numel() * workspace.element_size() < wsb:
        workspace = torch.empty(max(wsb, 16), dtype=torch.uint8, device=q.device)
    lib = load_library()
    ptrs = (q.data_ptr(), k.data_ptr(), v.data_ptr(), out.data_ptr(), lse.data_ptr(), dout.data_ptr(),
            dq.data_ptr(), dk.data_ptr(), dv.data_ptr(), B, H, L, d, int(w), int(dilation))
    tail = (_dtype_code(q), workspace.data_ptr(), workspace.numel() * workspace.element_size(),
            _stream(q.device))
    if dilated_heads is None:
        _check(lib.ft_winattn_bwd(*ptrs, *tail))
    else:
        _check(lib.ft_winattn_bwd_mixed(*ptrs, int(dilated_heads), *tail))
    return dq, dk, dv


def fwd_bwd(q, k, v, dout, w: int, dilation: int = 1, out=None, lse=None, dq=None, dk=None, dv=None,
            workspace: torch.Tensor | None = None):
    """Forward then backward in one call (ft_winattn_fwd_bwd; the recompute / checkpointing
    pattern): returns (out, lse, dq, dk, dv).  Inside the call the dQ kernel may read each lse
    row as the forward stores it."""
    _check_inputs(q, k, v, dout)
    B, H, L, d = q.shape
    out = torch.empty_like(q) if out is None else out
    lse = torch.empty((B, H, L), dtype=torch.float32, device=q.device) if lse is None else lse
    dq = torch.empty_like(q) if dq is None else dq
    dk = torch.empty_like(q) if dk is None else dk
    dv = torch.empty_like(q) if dv is None else dv
    wsb = workspace_bytes(q, w, dilation)
    if workspace is None or workspace.numel() * workspace.element_size() < wsb:
        workspace = torch.empty(max(wsb, 16), dtype=torch.uint8, device=q.device)
    _check(load_library().ft_winattn_fwd_bwd(
        q.data_ptr(), k.data_ptr(), v.data_ptr(), dout.data_ptr(), out.data_ptr(), lse.data_ptr(),
        dq.data_ptr(), dk.data_ptr(), dv.data_ptr(), B, H, L, d, int(w), int(dilation), _dtype_code(q),
        workspace.data_ptr(), workspace.numel() * workspace.element_size(), _stream(q.device)))
    return out, lse, dq, dk, dv


def tape_bytes(q: torch.Tensor, w: int) -> int:
    B, H, L, _ = q.shape
    return int(load_library().ft_winattn_tape_bytes(B, H, L, int(w)))


def fwd_tape(q, k, v, w: int, dilation: int = 1):
    """Forward that also materializes the band scores (ft_winattn_fwd_tape; band tensor-core
    kernels for bf16 where they apply, else CUDA-core kernels).  Returns (out, lse, tape) with
    tape fp32 [B, H, L, 2*min(w, L)+1]."""
    _check_inputs(q, k, v)
    B, H, L, d = q.shape
    out = torch.empty_like(q)
    lse = torch.empty((B, H, L), dtype=torch.float32, device=q.device)
    tape = torch.empty((B, H, L, 2 * min(int(w), L) + 1), dtype=torch.float32, device=q.device)
    _check(load_library().ft_winattn_fwd_tape(q.data_ptr(), k.data_ptr(), v.data_ptr(), out.data_ptr(),
                                              lse.data_ptr(), tape.data_ptr(), B, H, L, d, int(w),
                                              int(dilation), _dtype_code(q), _stream(q.device)))
    return out, lse, tape


def bwd_tape(q, k, v, out, lse, tape, dout, w: int, dilation: int = 1):
    """Backward reading the materialized scores instead of recomputing them (ft_winattn_bwd_tape)."""
    _check_inputs(q, k, v, out, dout)
    B, H, L, d = q.shape
    if tape.dtype != torch.float32 or not tape.is_contiguous() or \
            tape.numel() * 4 < tape_bytes(q, w):
        raise ValueError("tape must be the contiguous fp32 tensor fwd_tape returned")
    dq, dk, dv = torch.empty_like(q), torch.empty_like(q), torch.empty_like(q)
    wsb = workspace_bytes(q, w, dilation)
    ws = torch.empty(max(wsb, 16), dtype=torch.uint8, device=q.device)
    _check(load_library().ft_winattn_bwd_tape(
        q.data_ptr(), k.data_ptr(), v.data_ptr(), out.data_ptr(), lse.data_ptr(), tape.data_ptr(),
        dout.data_ptr(), dq.data_ptr(), dk.data_ptr(), dv.data_ptr(), B, H, L, d, int(w), int(dilation),
        _dtype_code(q), ws.data_ptr(), ws.numel(), _stream(q.device)))
    return dq, dk, dv


class WinAttn(torch.autograd.Function):
    """autograd wrapper: saves (q, k, v, out, lse); backward recomputes P from lse."""

    @staticmethod
    def forward(ctx, q, k, v, w: int, dilation: int = 1, dilated_heads: int | None = None):
        # the kernels take contiguous [B, H, L, d]: save the copies they read (a common layout,
        # x.view(B, L, H, d).transpose(1, 2), is not contiguous)
        q, k, v = q.contiguous(), k.contiguous(), v.contiguous()
        out, lse = fwd(q, k, v, w, dilation, dilated_heads=dilated_heads)
        ctx.save_for_backward(q, k, v, out, lse)
        ctx.w, ctx.dilation, ctx.dilated_heads = w, dilation, dilated_heads
        return out

    @staticmethod
    def backward(ctx, dout):
        q, k, v, out, lse = ctx.saved_tensors
        dq, dk, dv = bwd(q, k, v, out, lse, dout.contiguous(), ctx.w, ctx.dilation,
                         dilated_heads=ctx.dilated_heads)
        return dq, dk, dv, None, None, None


def win_attn(q, k, v, w: int, dilation: int = 1, dilated_heads: int | None = None):
    return WinAttn.apply(q, k, v, w, dilation, dilated_heads)
