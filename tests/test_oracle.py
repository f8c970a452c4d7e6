"""Pins for the fp64 oracle (oracle/), all CPU-only (-m "not gpu").

Every pin checks the oracle against something other than itself: hand-worked
golden examples, a dense band-masked numpy formulation, torch's fp64 SDPA and
autograd, closed forms, central finite differences, and gradient invariants.
Together they catch a dropped term, a wrong sign/index or transposed operand in
the oracle (each fails at least one test below).
"""
import json
import math
import os

import numpy as np
import pytest
import torch

import oracle
from synth import WinAttnShape, make_inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


# ----------------------------------------------------------------- independent references
def band_mask(L, w, dil):
    """Boolean [L, L] mask, M[i, j] = (j - i) = k*dil with |k| <= w (reading A4)."""
    i = np.arange(L)[:, None]
    j = np.arange(L)[None, :]
    diff = j - i
    return (diff % dil == 0) & (np.abs(diff) <= w * dil)


def dense_fwd(q, k, v, w, dil):
    """Dense fp64 attention with a band mask, in numpy matrix ops (independent code)."""
    L = q.shape[-2]
    M = band_mask(L, w, dil)
    S = np.einsum("bhid,bhjd->bhij", q, k)
    S = np.where(M, S, -np.inf)
    m = S.max(axis=-1, keepdims=True)
    E = np.exp(S - m)
    l = E.sum(axis=-1, keepdims=True)
    P = E / l
    return P @ v, (m + np.log(l))[..., 0], P


def torch_dense_grads(q, k, v, g, w, dil):
    L = q.shape[-2]
    M = torch.from_numpy(band_mask(L, w, dil))
    tq, tk, tv = (torch.tensor(x, dtype=torch.float64, requires_grad=True) for x in (q, k, v))
    S = torch.einsum("bhid,bhjd->bhij", tq, tk).masked_fill(~M, float("-inf"))
    O = torch.softmax(S, dim=-1) @ tv
    (O * torch.from_numpy(g)).sum().backward()
    return tq.grad.numpy(), tk.grad.numpy(), tv.grad.numpy()


def window_count_bruteforce(i, L, w, dil):
    return sum(1 for kk in range(-w, w + 1) if 0 <= i + kk * dil < L)


SMALL = [(1, 2, 64, 16, 4, 1), (2, 1, 64, 16, 4, 2), (1, 1, 37, 8, 5, 3), (1, 1, 20, 4, 0, 1),
         (1, 1, 20, 4, 30, 1), (1, 2, 33, 12, 7, 5)]


def _inputs(B, H, L, d, seed=0, scale=1.0):
    x = make_inputs(WinAttnShape(B, H, L, d, 0, 1), seed, "f32", q_scale=scale)
    return x["q64"], x["k64"], x["v64"], x["dout64"]


# ----------------------------------------------------------------- golden worked examples
def test_golden_worked_example_fwd_bwd():
    ex = json.load(open(os.path.join(GOLDEN, "worked_example_L3_w1.json")))
    sh = ex["shape"]
    q, k, v, g = (np.array(ex[n])[None, None] for n in ("q", "k", "v", "dout"))
    out, lse = oracle.fwd(q, k, v, sh["w"], sh["dilation"])
    np.testing.assert_allclose(out[0, 0], ex["out"], rtol=0, atol=1e-14)
    np.testing.assert_allclose(lse[0, 0], ex["lse"], rtol=0, atol=1e-14)
    dq, dk, dv = oracle.bwd(q, k, v, out, lse, g, sh["w"], sh["dilation"])
    np.testing.assert_allclose(dq[0, 0], ex["dq"], rtol=0, atol=1e-14)
    np.testing.assert_allclose(dk[0, 0], ex["dk"], rtol=0, atol=1e-14)
    np.testing.assert_allclose(dv[0, 0], ex["dv"], rtol=0, atol=1e-14)


def test_golden_worked_example_dilated():
    ex = json.load(open(os.path.join(GOLDEN, "worked_example_L5_w1_dil2.json")))
    sh = ex["shape"]
    q, k, v = (np.array(ex[n])[None, None] for n in ("q", "k", "v"))
    out, lse = oracle.fwd(q, k, v, sh["w"], sh["dilation"])
    np.testing.assert_allclose(out[0, 0], ex["out"], rtol=0, atol=1e-13)
    np.testing.assert_allclose(lse[0, 0], ex["lse"], rtol=0, atol=1e-14)


# ----------------------------------------------------------------- forward vs dense / library
@pytest.mark.parametrize("B,H,L,d,w,dil", SMALL)
def test_fwd_matches_dense_band_mask(B, H, L, d, w, dil):
    q, k, v, _ = _inputs(B, H, L, d, seed=L + d + w)
    out, lse = oracle.fwd(q, k, v, w, dil)
    O, LSE, _ = dense_fwd(q, k, v, w, dil)
    np.testing.assert_allclose(out, O, rtol=1e-12, atol=1e-13)
    np.testing.assert_allclose(lse, LSE, rtol=1e-12, atol=1e-13)


@pytest.mark.parametrize("B,H,L,d,w,dil", SMALL)
def test_fwd_matches_torch_sdpa_fp64(B, H, L, d, w, dil):
    q, k, v, _ = _inputs(B, H, L, d, seed=7)
    out, _ = oracle.fwd(q, k, v, w, dil)
    M = torch.from_numpy(band_mask(L, w, dil))
    ref = torch.nn.functional.scaled_dot_product_attention(
        torch.from_numpy(q), torch.from_numpy(k), torch.from_numpy(v), attn_mask=M, scale=1.0)
    np.testing.assert_allclose(out, ref.numpy(), rtol=1e-12, atol=1e-13)


def test_full_attention_when_window_covers_sequence():
    """w >= L-1, dilation 1 => ordinary softmax attention (library routine, no mask)."""
    q, k, v, _ = _inputs(1, 2, 29, 8, seed=3)
    for w in (28, 29, 1000):
        out, lse = oracle.fwd(q, k, v, w, 1)
        ref = torch.nn.functional.scaled_dot_product_attention(
            torch.from_numpy(q), torch.from_numpy(k), torch.from_numpy(v), scale=1.0)
        np.testing.assert_allclose(out, ref.numpy(), rtol=1e-12, atol=1e-13)
        lse_ref = torch.logsumexp(torch.from_numpy(q) @ torch.from_numpy(k).transpose(-1, -2), -1)
        np.testing.assert_allclose(lse, lse_ref.numpy(), rtol=1e-13, atol=1e-13)


def test_overflow_probe_q_times_16():
    """Logits ~ x16: the max-subtraction keeps everything finite."""
    q, k, v, _ = _inputs(1, 1, 64, 16, seed=11, scale=16.0)
    out, lse = oracle.fwd(q, k, v, 4, 1)
    assert np.isfinite(out).all() and np.isfinite(lse).all()
    O, LSE, _ = dense_fwd(q, k, v, 4, 1)
    np.testing.assert_allclose(out, O, rtol=1e-12, atol=1e-12)
    np.testing.assert_allclose(lse, LSE, rtol=1e-13)


# ----------------------------------------------------------------- closed forms
def test_window_count_closed_form():
    """|N(i)| = min(w, floor(i/dil)) + min(w, floor((L-1-i)/dil)) + 1 vs brute force."""
    for L in (1, 2, 7, 33):
        for w in (0, 1, 3, 40):
            for dil in (1, 2, 3, 8):
                for i in range(L):
                    cf = min(w, i // dil) + min(w, (L - 1 - i) // dil) + 1
                    assert cf == window_count_bruteforce(i, L, w, dil)


@pytest.mark.parametrize("L,w,dil", [(64, 4, 1), (37, 5, 3), (50, 7, 2), (16, 100, 1), (1, 3, 1)])
def test_q_zero_closed_form(L, w, dil):
    """q = 0 => all logits 0 => lse_i = ln|N(i)| and o_i = mean of v over N(i) (boundary count, A2)."""
    _, k, v, _ = _inputs(1, 1, L, 8, seed=5)
    q = np.zeros_like(k)
    out, lse = oracle.fwd(q, k, v, w, dil)
    for i in range(L):
        idx = [i + kk * dil for kk in range(-w, w + 1) if 0 <= i + kk * dil < L]
        assert lse[0, 0, i] == pytest.approx(math.log(len(idx)), abs=1e-14)
        np.testing.assert_allclose(out[0, 0, i], v[0, 0, idx].mean(axis=0), rtol=1e-13, atol=1e-14)


def test_w_zero_closed_form():
    """w = 0 => o = v, lse_i = q_i.k_i, dq = dk = 0, dv = dout."""
    q, k, v, g = _inputs(1, 2, 20, 4, seed=9)
    out, lse = oracle.fwd(q, k, v, 0, 1)
    np.testing.assert_array_equal(out, v)
    np.testing.assert_allclose(lse, (q * k).sum(-1), rtol=1e-15, atol=1e-15)
    dq, dk, dv = oracle.bwd(q, k, v, out, lse, g, 0, 1)
    np.testing.assert_allclose(dq, 0.0, atol=1e-15)
    np.testing.assert_allclose(dk, 0.0, atol=1e-15)
    np.testing.assert_array_equal(dv, g)


@pytest.mark.parametrize("L,w,dil", [(64, 4, 2), (37, 5, 3), (41, 3, 4)])
def test_dilation_is_residue_decomposition(L, w, dil):
    """Dilation dil == dil independent dilation-1 problems on x[r::dil] (reading A4)."""
    q, k, v, g = _inputs(1, 1, L, 8, seed=L)
    out, lse = oracle.fwd(q, k, v, w, dil)
    dq, dk, dv = oracle.bwd(q, k, v, out, lse, g, w, dil)
    for r in range(dil):
        s = np.s_[..., r::dil, :]
        o_r, l_r = oracle.fwd(q[s], k[s], v[s], w, 1)
        np.testing.assert_array_equal(out[s], o_r)
        np.testing.assert_array_equal(lse[..., r::dil], l_r)
        dq_r, dk_r, dv_r = oracle.bwd(q[s], k[s], v[s], o_r, l_r, g[s], w, 1)
        np.testing.assert_array_equal(dq[s], dq_r)
        np.testing.assert_array_equal(dk[s], dk_r)
        np.testing.assert_array_equal(dv[s], dv_r)


def test_rows_of_softmax_sum_to_one():
    """v = 1 => o = sum_j P_ij = 1 for every row."""
    q, k, _, _ = _inputs(1, 2, 50, 8, seed=4, scale=3.0)
    for w, dil in ((4, 1), (3, 3), (60, 1)):
        out, _ = oracle.fwd(q, k, np.ones_like(k), w, dil)
        np.testing.assert_allclose(out, 1.0, rtol=0, atol=1e-14)


# ----------------------------------------------------------------- backward
@pytest.mark.parametrize("B,H,L,d,w,dil", SMALL)
def test_bwd_matches_torch_autograd(B, H, L, d, w, dil):
    q, k, v, g = _inputs(B, H, L, d, seed=100 + L)
    out, lse = oracle.fwd(q, k, v, w, dil)
    dq, dk, dv = oracle.bwd(q, k, v, out, lse, g, w, dil)
    rq, rk, rv = torch_dense_grads(q, k, v, g, w, dil)
    for a, b in ((dq, rq), (dk, rk), (dv, rv)):
        np.testing.assert_allclose(a, b, rtol=1e-11, atol=1e-12)


def test_bwd_dout_ones_is_grad_of_sum():
    """JAX/Julia seed the gradient with sum(outputs), i.e. dout = 1."""
    q, k, v, _ = _inputs(1, 1, 40, 8, seed=21)
    g = np.ones_like(q)
    out, lse = oracle.fwd(q, k, v, 5, 2)
    dq, dk, dv = oracle.bwd(q, k, v, out, lse, g, 5, 2)
    rq, rk, rv = torch_dense_grads(q, k, v, g, 5, 2)
    for a, b in ((dq, rq), (dk, rk), (dv, rv)):
        np.testing.assert_allclose(a, b, rtol=1e-11, atol=1e-12)


def test_bwd_central_finite_differences_C1():
    """Central FD of L = sum(G o O) w.r.t. every element of q, k, v at C1 (h = 1e-6)."""
    B, H, L, d, w = 1, 1, 64, 16, 4
    for dil in (1, 3):
        q, k, v, g = _inputs(B, H, L, d, seed=0)
        out, lse = oracle.fwd(q, k, v, w, dil)
        grads = oracle.bwd(q, k, v, out, lse, g, w, dil)
        h = 1e-6
        for which in range(3):
            xs = [q.copy(), k.copy(), v.copy()]
            fd = np.empty_like(xs[which])
            flat = xs[which].reshape(-1)
            for e in range(flat.size):
                orig = flat[e]
                flat[e] = orig + h
                lp = (oracle.fwd(*xs, w, dil)[0] * g).sum()
                flat[e] = orig - h
                lm = (oracle.fwd(*xs, w, dil)[0] * g).sum()
                flat[e] = orig
                fd.reshape(-1)[e] = (lp - lm) / (2 * h)
            an = grads[which]
            tol = 1e-6 * np.abs(an).max() + 1e-8
            assert np.abs(fd - an).max() <= tol, (which, dil, np.abs(fd - an).max())


@pytest.mark.parametrize("w,dil", [(4, 1), (6, 2), (50, 1)])
def test_bwd_invariants(w, dil):
    q, k, v, g = _inputs(2, 2, 48, 8, seed=w * 10 + dil)
    out, lse = oracle.fwd(q, k, v, w, dil)
    dq, dk, dv = oracle.bwd(q, k, v, out, lse, g, w, dil)
    # sum_j dS_ij = 0 for each i  =>  sum_j dk_j = 0 (per unit, per feature)
    np.testing.assert_allclose(dk.sum(axis=2), 0.0, atol=1e-12)
    # sum_j P_ij = 1  =>  sum_j dv_j = sum_i dout_i
    np.testing.assert_allclose(dv.sum(axis=2), g.sum(axis=2), rtol=1e-12, atol=1e-12)
    # sum_i q_i.dq_i = sum_ij dS_ij S_ij = sum_j k_j.dk_j
    np.testing.assert_allclose((q * dq).sum(axis=(2, 3)), (k * dk).sum(axis=(2, 3)),
                               rtol=1e-11, atol=1e-11)


# ----------------------------------------------------------------- sampled (row) entry points
@pytest.mark.parametrize("w,dil", [(4, 1), (5, 3), (40, 1)])
def test_row_entry_points_match_full(w, dil):
    q, k, v, g = _inputs(2, 1, 45, 8, seed=31)
    out, lse = oracle.fwd(q, k, v, w, dil)
    dq, dk, dv = oracle.bwd(q, k, v, out, lse, g, w, dil)
    rows = np.array([0, 1, 7, 44, 45, 60, 89])
    o_r, l_r = oracle.fwd_rows(q, k, v, w, dil, rows)
    np.testing.assert_allclose(o_r, out.reshape(-1, 8)[rows], rtol=1e-13, atol=1e-14)
    np.testing.assert_allclose(l_r, lse.reshape(-1)[rows], rtol=1e-14, atol=1e-14)
    dq_r, dk_r, dv_r = oracle.bwd_rows(q, k, v, g, w, dil, rows)
    np.testing.assert_allclose(dq_r, dq.reshape(-1, 8)[rows], rtol=1e-11, atol=1e-13)
    np.testing.assert_allclose(dk_r, dk.reshape(-1, 8)[rows], rtol=1e-11, atol=1e-13)
    np.testing.assert_allclose(dv_r, dv.reshape(-1, 8)[rows], rtol=1e-11, atol=1e-13)
