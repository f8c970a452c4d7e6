"""fp64 CPU oracle for banded (dilated) window attention — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_pldi_tangzwjzyz22_b200``) never imports it and shares no code with it.

The arithmetic lives in ``winattn_ref.c`` (plain C loop nests following PAPER.md
Fig. 8 / Fig. 10, lines 215-231 and 306-321); this module only compiles it with gcc
(``-O2 -fopenmp``, no fast-math) and marshals numpy fp64 arrays through ctypes.

Pins (tests/test_oracle.py, ``-m "not gpu"``): dense band-masked numpy attention,
torch fp64 SDPA, torch.autograd, central finite differences, a hand-worked golden
example (tests/golden/), closed forms (w=0, q=0, w>=L-1, dilation = residue
decomposition), and gradient invariants.  Every function below is pinned.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "winattn_ref.c")
_HDR = os.path.join(_HERE, "winattn_ref.h")
_LIB_PATH = os.path.join(_HERE, "libwinattn_ref.so")
_lock = threading.Lock()
_lib = None

_i64 = ctypes.c_int64
_dp = ctypes.POINTER(ctypes.c_double)
_ip = ctypes.POINTER(ctypes.c_int64)


def build(force: bool = False) -> str:
    """Compile the oracle shared library with gcc (fp64, -O2, OpenMP, no fast-math)."""
    newest_src = max(os.path.getmtime(_SRC), os.path.getmtime(_HDR))
    if force or not os.path.exists(_LIB_PATH) or os.path.getmtime(_LIB_PATH) < newest_src:
        tmp = _LIB_PATH + f".tmp{os.getpid()}"
        cmd = ["gcc", "-O2", "-fno-fast-math", "-fopenmp", "-fPIC", "-shared", "-std=c99",
               "-o", tmp, _SRC, "-lm"]
        subprocess.run(cmd, check=True)
        os.replace(tmp, _LIB_PATH)
    return _LIB_PATH


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB_PATH)
            lib.ref_num_threads.restype = ctypes.c_int
            lib.ref_set_num_threads.argtypes = [ctypes.c_int]
            lib.ref_winattn_fwd.argtypes = [_dp, _dp, _dp, _dp, _dp, _i64, _i64, _i64, _i64, _i64]
            lib.ref_winattn_bwd.argtypes = [_dp] * 9 + [_i64] * 5
            lib.ref_winattn_fwd_rows.argtypes = [_dp, _dp, _dp] + [_i64] * 5 + [_ip, _i64, _dp, _dp]
            lib.ref_winattn_bwd_rows.argtypes = [_dp] * 4 + [_i64] * 5 + [_ip, _i64, _dp, _dp, _dp]
            _lib = lib
    return _lib


def _f64(x) -> np.ndarray:
    a = np.ascontiguousarray(np.asarray(x, dtype=np.float64))
    return a


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(_dp)


def num_threads() -> int:
    return int(_load().ref_num_threads())


def set_num_threads(n: int) -> None:
    _load().ref_set_num_threads(int(n))


def _dims(q):
    if q.ndim != 4:
        raise ValueError("expected [B, H, L, d]")
    B, H, L, d = q.shape
    return B * H, L, d


def fwd(q, k, v, w: int, dilation: int = 1):
    """(out, lse) in fp64 for inputs [B, H, L, d]; lse is [B, H, L]."""
    q, k, v = _f64(q), _f64(k), _f64(v)
    units, L, d = _dims(q)
    out = np.empty_like(q)
    lse = np.empty(q.shape[:3], dtype=np.float64)
    _load().ref_winattn_fwd(_ptr(q), _ptr(k), _ptr(v), _ptr(out), _ptr(lse),
                            units, L, d, int(w), int(dilation))
    return out, lse


def bwd(q, k, v, out, lse, dout, w: int, dilation: int = 1):
    """(dq, dk, dv) in fp64 given the forward's out and lse."""
    q, k, v, out, lse, dout = (_f64(x) for x in (q, k, v, out, lse, dout))
    units, L, d = _dims(q)
    dq, dk, dv = np.empty_like(q), np.empty_like(q), np.empty_like(q)
    _load().ref_winattn_bwd(_ptr(q), _ptr(k), _ptr(v), _ptr(out), _ptr(lse), _ptr(dout),
                            _ptr(dq), _ptr(dk), _ptr(dv), units, L, d, int(w), int(dilation))
    return dq, dk, dv


def fwd_rows(q, k, v, w: int, dilation: int, rows):
    """Sampled forward: ``rows`` are flat ids u*L + i.  Returns (out [n,d], lse [n])."""
    q, k, v = _f64(q), _f64(k), _f64(v)
    units, L, d = _dims(q)
    rows = np.ascontiguousarray(np.asarray(rows, dtype=np.int64))
    n = rows.shape[0]
    out = np.empty((n, d), dtype=np.float64)
    lse = np.empty((n,), dtype=np.float64)
    _load().ref_winattn_fwd_rows(_ptr(q), _ptr(k), _ptr(v), units, L, d, int(w), int(dilation),
                                 rows.ctypes.data_as(_ip), n, _ptr(out), _ptr(lse))
    return out, lse


def bwd_rows(q, k, v, dout, w: int, dilation: int, rows):
    """Sampled backward from scratch (own lse/o/D): returns (dq, dk, dv), each [n, d]."""
    q, k, v, dout = (_f64(x) for x in (q, k, v, dout))
    units, L, d = _dims(q)
    rows = np.ascontiguousarray(np.asarray(rows, dtype=np.int64))
    n = rows.shape[0]
    dq, dk, dv = (np.empty((n, d), dtype=np.float64) for _ in range(3))
    _load().ref_winattn_bwd_rows(_ptr(q), _ptr(k), _ptr(v), _ptr(dout), units, L, d, int(w),
                                 int(dilation), rows.ctypes.data_as(_ip), n,
                                 _ptr(dq), _ptr(dk), _ptr(dv))
    return dq, dk, dv
