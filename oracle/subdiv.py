"""fp64 CPU oracle of SubdivNet's circular difference — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__`` and the bench tools may import it; the product path never
does and shares no code with it.  The arithmetic is ``subdiv_ref.c`` (plain loops following
PAPER.md Fig. 2, lines 89-119); this module compiles it with gcc (-O2, no fast-math) and passes
numpy arrays through ctypes.  Pins: tests/test_oracle_subdiv.py (the operator formulation of
Fig. 2(c) in numpy and torch, torch.autograd, a hand-worked golden example, invariants, central
finite differences).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "subdiv_ref.c")
_LIB = os.path.join(_HERE, "libsubdiv_ref.so")
_lock = threading.Lock()
_lib = None
_dp = ctypes.POINTER(ctypes.c_double)
_ip = ctypes.POINTER(ctypes.c_int64)


def build(force: bool = False) -> str:
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.run(["gcc", "-O2", "-fno-fast-math", "-fPIC", "-shared", "-std=c99", "-o", tmp, _SRC,
                        "-lm"], check=True)
        os.replace(tmp, _LIB)
    return _LIB


def _load():
    global _lib
    with _lock:
        if _lib is None:
            build()
            lib = ctypes.CDLL(_LIB)
            lib.ref_subdiv_fwd.argtypes = [_dp, _ip, _dp, ctypes.c_int64, ctypes.c_int64]
            lib.ref_subdiv_bwd.argtypes = [_dp, _ip, _dp, _dp, ctypes.c_int64, ctypes.c_int64]
            _lib = lib
    return _lib


def _prep(e, adj):
    e = np.ascontiguousarray(e, dtype=np.float64)
    adj = np.ascontiguousarray(adj, dtype=np.int64)
    assert e.ndim == 2 and adj.shape == (e.shape[0], 3)
    return e, adj


def fwd(e, adj):
    """y [n_faces, n_feats] = sum_j |e[adj[i, j]] - e[adj[i, (j+1) % 3]]| (Fig. 2)."""
    e, adj = _prep(e, adj)
    y = np.empty_like(e)
    _load().ref_subdiv_fwd(e.ctypes.data_as(_dp), adj.ctypes.data_as(_ip), y.ctypes.data_as(_dp),
                           e.shape[0], e.shape[1])
    return y


def bwd(e, adj, dy):
    """de for the loss sum(y * dy), with sign(0) = 0 (reading S1)."""
    e, adj = _prep(e, adj)
    dy = np.ascontiguousarray(dy, dtype=np.float64)
    de = np.empty_like(e)
    _load().ref_subdiv_bwd(e.ctypes.data_as(_dp), adj.ctypes.data_as(_ip), dy.ctypes.data_as(_dp),
                           de.ctypes.data_as(_dp), e.shape[0], e.shape[1])
    return de
