"""C-ABI checks that need no GPU: the library builds for sm_100a, loads, exports every
symbol include/ft_winattn.h declares, and argument validation returns the documented
status codes before any launch (fake device pointers are never dereferenced)."""
from __future__ import annotations

import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_pldi_tangzwjzyz22_b200 as ft

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ft_winattn.h")
HEADERS = [os.path.join(ROOT, "include", h) for h in sorted(os.listdir(os.path.join(ROOT, "include")))
           if h.endswith(".h")]

OK, INVALID, NOTSUP, MISALIGNED = 0, 1, 2, 3


@pytest.fixture(scope="module")
def lib():
    return ft.load_library(build_if_missing=True)


def declared_symbols():
    src = "\n".join(open(h).read() for h in HEADERS)
    return sorted(set(re.findall(r"^\S[^;()]*?\b(ft_\w+)\s*\(", src, flags=re.M)))


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for s in ("ft_winattn_fwd", "ft_winattn_bwd", "ft_winattn_fwd_bwd", "ft_winattn_bwd_workspace_bytes",
              "ft_winattn_plan", "ft_status_str", "ft_winattn_abi_version"):
        assert s in syms


def test_library_exports_every_declared_symbol(lib):
    out = subprocess.run(["nm", "-D", "--defined-only", ft.lib_path()], capture_output=True,
                         text=True, check=True).stdout
    exported = set(re.findall(r"\bT\s+(\w+)", out))
    missing = [s for s in declared_symbols() if s not in exported]
    assert not missing, missing
    assert lib.ft_winattn_abi_version() == 2


def test_library_is_sm100a(lib):
    out = subprocess.run(["cuobjdump", "--list-elf", ft.lib_path()], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_library_has_tcgen05_and_tma(lib):
    sass = subprocess.run(["cuobjdump", "-sass", ft.lib_path()], capture_output=True,
                          text=True).stdout
    assert "UTCHMMA" in sass          # tcgen05.mma
    assert "UTMALDG" in sass          # TMA load
    assert "LDTM" in sass             # tcgen05.ld


# fake, 16-byte aligned "device" pointers in disjoint ranges (never dereferenced)
def P(i, off=0):
    return ctypes.c_void_p(0x10000000000 + i * 0x100000000 + off)


def fwd_call(lib, q=None, k=None, v=None, out=None, lse=None, B=1, H=1, L=64, d=64, w=4, dil=1,
             dt=1, alias=None):
    given = [q, k, v, out, lse]
    args = [P(i) if a is None else a for i, a in enumerate(given)]
    if alias:
        args[alias[0]] = args[alias[1]]
    return lib.ft_winattn_fwd(*args, B, H, L, d, w, dil, dt, None)


def test_fwd_validation(lib):
    assert fwd_call(lib, q=ctypes.c_void_p(0)) == INVALID
    assert fwd_call(lib, B=0) == INVALID
    assert fwd_call(lib, L=0) == INVALID
    assert fwd_call(lib, w=-1) == INVALID
    assert fwd_call(lib, dil=0) == INVALID
    assert fwd_call(lib, d=24) == NOTSUP
    assert fwd_call(lib, d=528) == NOTSUP
    assert fwd_call(lib, dt=7) == NOTSUP
    assert fwd_call(lib, q=P(0, 8)) == MISALIGNED
    assert fwd_call(lib, alias=(3, 0)) == INVALID     # out aliases q
    assert fwd_call(lib, alias=(4, 3)) == INVALID     # lse aliases out


def bwd_call(lib, ws_bytes=None, ws=None, alias=None, **kw):
    B, H, L, d, w, dil, dt = (kw.get(n, dv) for n, dv in
                              (("B", 1), ("H", 1), ("L", 64), ("d", 64), ("w", 4), ("dil", 1), ("dt", 1)))
    need = lib.ft_winattn_bwd_workspace_bytes(B, H, L, d, w, dil, dt)
    args = [P(i) for i in range(9)]
    if alias:
        args[alias[0]] = args[alias[1]]
    return lib.ft_winattn_bwd(*args, B, H, L, d, w, dil, dt, ws or P(9),
                              need if ws_bytes is None else ws_bytes, None)


def test_bwd_validation(lib):
    assert bwd_call(lib, w=-2) == INVALID
    assert bwd_call(lib, ws_bytes=0) == INVALID          # workspace too small
    assert bwd_call(lib, ws=P(9, 4)) == MISALIGNED
    assert bwd_call(lib, alias=(6, 0)) == INVALID        # dq aliases q
    assert bwd_call(lib, alias=(7, 6)) == INVALID        # dk aliases dq
    assert bwd_call(lib, d=8) == NOTSUP


def fwd_bwd_call(lib, alias=None, B=1, H=1, L=64, d=64, w=4, dil=1, dt=1, ws_bytes=None):
    """ft_winattn_fwd_bwd(q, k, v, dout, out, lse, dq, dk, dv, ..., workspace, bytes, stream)"""
    need = lib.ft_winattn_bwd_workspace_bytes(B, H, L, d, w, dil, dt)
    args = [P(i) for i in range(9)]
    if alias:
        args[alias[0]] = args[alias[1]]
    return lib.ft_winattn_fwd_bwd(*args, B, H, L, d, w, dil, dt, P(9),
                                  need if ws_bytes is None else ws_bytes, None)


def test_fwd_bwd_validation(lib):
    """the combined call rejects what either half rejects, and also dout overlapping out / lse
    (out and lse are outputs of the call)"""
    assert fwd_bwd_call(lib, w=-1) == INVALID
    assert fwd_bwd_call(lib, ws_bytes=0) == INVALID
    assert fwd_bwd_call(lib, alias=(4, 3)) == INVALID    # out aliases dout
    assert fwd_bwd_call(lib, alias=(5, 3)) == INVALID    # lse aliases dout
    assert fwd_bwd_call(lib, alias=(4, 0)) == INVALID    # out aliases q
    assert fwd_bwd_call(lib, alias=(6, 4)) == INVALID    # dq aliases out
    assert fwd_bwd_call(lib, alias=(8, 5)) == INVALID    # dv aliases lse
    assert fwd_bwd_call(lib, d=24) == NOTSUP
    bad = [P(i) for i in range(9)]
    bad[3] = P(3, 8)
    need = lib.ft_winattn_bwd_workspace_bytes(1, 1, 64, 64, 4, 1, 1)
    assert lib.ft_winattn_fwd_bwd(*bad, 1, 1, 64, 64, 4, 1, 1, P(9), need, None) == MISALIGNED


def test_debug_knobs(lib):
    """ft_winattn_debug_set / get: documented knobs and values only; plan() follows the path knob"""
    assert lib.ft_winattn_debug_set(7, 1) == INVALID
    assert lib.ft_winattn_debug_set(0, 3) == INVALID
    assert lib.ft_winattn_debug_set(1, 2) == INVALID
    assert lib.ft_winattn_debug_get(9) == -1
    with ft.knobs(path="simt"):
        assert ft.debug_get("path") == 1
        assert ft.plan(False, 1, 8, 10000, 512, 32, 1, ft.FT_BF16)[0] == ft.PATH_SIMT
    with ft.knobs(path="tc"):
        with pytest.raises(ft.FtError):   # no tensor-core kernel for d = 48
            ft.plan(False, 1, 1, 300, 48, 4, 1, ft.FT_BF16)
    assert ft.debug_get("path") == 0
    with ft.knobs(narrow=0, pdl=0):
        assert ft.debug_get("narrow") == 0 and ft.debug_get("pdl") == 0
    assert ft.debug_get("narrow") == 1 and ft.debug_get("pdl") == 1
    # dS tape knob: 0 off, 1 where it pays (default), 2 forced; nothing else
    assert lib.ft_winattn_debug_set(5, 3) == INVALID
    assert ft.debug_get("dstape") == 1
    with ft.knobs(dstape=2):
        assert ft.debug_get("dstape") == 2


def test_workspace_dstape_layout(lib):
    """The backward workspace (include/ft_winattn.h): D (fp32 per row) always; the dS tape regions
    -- a flag word per row and two fp32 planes of tsw = 4 ceil((2w + 4) / 4) floats per row, each
    region rounded up to 256 bytes -- exactly where the tensor-core kernels use the tape (fp32
    d >= 256, bf16 band kernels d > 256; any d they support with the knob at 2)."""
    r256 = lambda x: (x + 255) // 256 * 256
    def ws(B, H, L, d, w, dil, dt):
        return lib.ft_winattn_bwd_workspace_bytes(B, H, L, d, w, dil, dt)
    F32, BF16 = ft.FT_F32, ft.FT_BF16
    rows = 2 * 3 * 1000
    tape = lambda w: r256(rows * 4) + r256(rows * 4) + 2 * r256(rows * 4 * ((2 * w + 4 + 3) // 4 * 4))
    assert ws(2, 3, 1000, 512, 32, 1, F32) == tape(32)        # fp32, d >= 256
    assert ws(2, 3, 1000, 256, 5, 3, F32) == tape(5)
    assert ws(2, 3, 1000, 128, 32, 1, F32) == r256(rows * 4)  # fp32 d = 128: recompute
    assert ws(2, 3, 1000, 512, 32, 1, BF16) == tape(32)       # bf16 band kernels, d > 256
    assert ws(2, 3, 1000, 256, 32, 1, BF16) == r256(rows * 4) # bf16 d = 256: recompute
    assert ws(2, 3, 1000, 512, 100, 1, F32) == r256(rows * 4) # w > 32: CUDA-core fp32 path
    assert ws(2, 3, 1000, 512, 100, 1, BF16) == r256(rows * 4) # w > 64: chunked kernels
    with ft.knobs(dstape=2):
        assert ws(2, 3, 1000, 256, 32, 1, BF16) == tape(32)
    with ft.knobs(dstape=0):   # knob 0 keeps the size (the call then ignores the tape regions)
        assert ws(2, 3, 1000, 512, 32, 1, F32) == tape(32)


def test_workspace_and_plan(lib):
    assert lib.ft_winattn_bwd_workspace_bytes(2, 3, 100, 64, 4, 1, 1) >= 2 * 3 * 100 * 4
    assert lib.ft_winattn_bwd_workspace_bytes(0, 3, 100, 64, 4, 1, 1) == 0
    path, n = ft.plan(False, 1, 8, 10000, 512, 32, 1, ft.FT_BF16)
    assert path == ft.PATH_TC and n == 1
    path, n = ft.plan(False, 1, 8, 10000, 512, 32, 1, ft.FT_F32)   # fp32 tensor-core kernels
    assert path == ft.PATH_TC and n == 1
    path, n = ft.plan(True, 1, 8, 10000, 512, 32, 1, ft.FT_F32)
    assert path == ft.PATH_TC and n == 2
    path, n = ft.plan(False, 1, 8, 4096, 64, 256, 1, ft.FT_F32)    # w > 32, d = 64: WIDE sub-bands
    assert path == ft.PATH_TC and n == 1
    path, n = ft.plan(True, 1, 8, 4096, 64, 256, 1, ft.FT_F32)     # D = dout . out, dQ, dK / dV
    assert path == ft.PATH_TC and n == 3
    path, n = ft.plan(False, 1, 8, 4096, 128, 256, 1, ft.FT_F32)   # w > 32, d = 128: 128-row steps
    assert path == ft.PATH_TC
    path, n = ft.plan(False, 1, 8, 4096, 192, 256, 1, ft.FT_F32)   # w > 32, d not in {64, 128}: CUDA cores
    assert path == ft.PATH_SIMT
    path, n = ft.plan(True, 1, 1, 64, 16, 4, 1, ft.FT_F32)
    assert path == ft.PATH_SIMT and n >= 1
    with pytest.raises(ft.FtError):
        ft.plan(False, 1, 1, 64, 24, 4, 1, ft.FT_F32)


def test_status_strings(lib):
    for s in range(5):
        assert lib.ft_status_str(s)
    assert b"INVALID" in lib.ft_status_str(1)


def test_mixed_validation(lib):
    """ft_winattn_fwd_mixed / bwd_mixed: dilated_heads outside [0, heads] and every check of the
    plain entry points fail before any launch (fake pointers are never dereferenced)."""
    args = [P(i) for i in range(5)]
    assert lib.ft_winattn_fwd_mixed(*args, 1, 4, 64, 64, 4, 2, 5, 1, None) == INVALID
    assert lib.ft_winattn_fwd_mixed(*args, 1, 4, 64, 64, 4, 2, -1, 1, None) == INVALID
    assert lib.ft_winattn_fwd_mixed(*args, 1, 4, 64, 64, 4, 0, 2, 1, None) == INVALID   # dilation 0
    assert lib.ft_winattn_fwd_mixed(*args, 1, 4, 64, 24, 4, 2, 2, 1, None) == NOTSUP    # d = 24
    bad = list(args)
    bad[0] = P(0, 8)
    assert lib.ft_winattn_fwd_mixed(*bad, 1, 4, 64, 64, 4, 2, 2, 1, None) == MISALIGNED
    need = lib.ft_winattn_bwd_workspace_bytes(1, 4, 64, 64, 4, 2, 1)
    b = [P(i) for i in range(9)]
    assert lib.ft_winattn_bwd_mixed(*b, 1, 4, 64, 64, 4, 2, 7, 1, P(9), need, None) == INVALID
    assert lib.ft_winattn_bwd_mixed(*b, 1, 4, 64, 64, 4, 2, 2, 1, P(9), 0, None) == INVALID
    b[7] = b[6]                                                                          # dk aliases dq
    assert lib.ft_winattn_bwd_mixed(*b, 1, 4, 64, 64, 4, 2, 2, 1, P(9), need, None) == INVALID


def test_tape_validation(lib):
    assert lib.ft_winattn_tape_bytes(2, 3, 100, 4) == 2 * 3 * 100 * 9 * 4
    assert lib.ft_winattn_tape_bytes(1, 1, 10, 50) == 10 * 21 * 4      # w clamped to L
    assert lib.ft_winattn_tape_bytes(0, 1, 10, 5) == 0
    a = [P(i) for i in range(5)]
    assert lib.ft_winattn_fwd_tape(*a, None, 1, 1, 64, 64, 4, 1, 1, None) == INVALID
    assert lib.ft_winattn_fwd_tape(*a, P(5, 4), 1, 1, 64, 64, 4, 1, 1, None) == MISALIGNED
    assert lib.ft_winattn_fwd_tape(*a, P(5), 1, 1, 64, 24, 4, 1, 1, None) == NOTSUP
    need = lib.ft_winattn_bwd_workspace_bytes(1, 1, 64, 64, 4, 1, 1)
    b = [P(i) for i in range(10)]
    assert lib.ft_winattn_bwd_tape(*b[:5], None, *b[6:10], 1, 1, 64, 64, 4, 1, 1, P(11), need, None) == INVALID
    assert lib.ft_winattn_bwd_tape(*b, 1, 1, 64, 64, 4, 1, 1, P(11), 0, None) == INVALID


def test_subdiv_validation(lib):
    """SubdivNet circular difference (include/ft_subdiv.h): argument checks before any launch."""
    f = lib.ft_subdiv_circdiff_fwd
    f.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int64, ctypes.c_int64,
                  ctypes.c_int, ctypes.c_void_p]
    assert f(None, P(1), P(2), 100, 64, 0, None) == INVALID
    assert f(P(0), P(1), P(2), 0, 64, 0, None) == INVALID
    assert f(P(0), P(1), P(2), 100, 64, 5, None) == NOTSUP
    assert f(P(0, 8), P(1), P(2), 100, 64, 0, None) == MISALIGNED
    assert f(P(0), P(1, 2), P(2), 100, 64, 0, None) == MISALIGNED
    assert f(P(0), P(1), P(0), 100, 64, 0, None) == INVALID           # y aliases e
    b = lib.ft_subdiv_circdiff_bwd
    b.argtypes = [ctypes.c_void_p] * 4 + [ctypes.c_int64, ctypes.c_int64, ctypes.c_int, ctypes.c_int,
                                          ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p]
    lib.ft_subdiv_circdiff_bwd_workspace_bytes.restype = ctypes.c_size_t
    lib.ft_subdiv_circdiff_bwd_workspace_bytes.argtypes = [ctypes.c_int64, ctypes.c_int64, ctypes.c_int]
    assert lib.ft_subdiv_circdiff_bwd_workspace_bytes(100, 64, 0) == 0
    need = lib.ft_subdiv_circdiff_bwd_workspace_bytes(100, 64, 1)
    assert need >= 100 * 64 * 4
    assert b(P(0), P(1), P(2), P(3), 100, 64, 1, 0, P(4), 0, None) == INVALID     # workspace too small
    assert b(P(0), P(1), P(2), P(2), 100, 64, 0, 0, None, 0, None) == INVALID     # de aliases dy
    assert b(P(0), P(1), P(2), P(3, 4), 100, 64, 0, 1, None, 0, None) == MISALIGNED
