"""Tape vs recompute on B200 (Fig. 18): the paper's
selective materialization decides per intermediate whether the gradient program reads it from a
tape or recomputes it.  Here the intermediate is the band score s_ij = q_i . k_j (Fig. 8's `dot`):

  recompute : ft_winattn_fwd + ft_winattn_bwd (saves lse only; bwd reruns the score GEMM)
  tape      : ft_winattn_fwd_tape + ft_winattn_bwd_tape (fwd also writes s, fp32 [rows][2w+1];
              bwd reads it and skips the score GEMM)

on the band tensor-core kernels (bf16; the d = 64, w <= 32 narrow kernels are switched off for
the recompute leg so both legs use the same kernels) and on the CUDA-core kernels (fp32).  Both
legs of one family run on the same inputs; one JSON line per case with ms per fwd+bwd step (CUDA
events, mean of 20 after 3 warm-ups, L2 flushed between steps) and the tape's extra HBM bytes per
step (one write + two reads, the dQ and dK/dV kernels each read it).

The second table is the dS tape between the two fp32 tensor-core backward kernels
(FT_KNOB_DSTAPE): the dQ kernel stores P and dS of every band entry and the dK/dV kernel reads them
instead of recomputing S^T and dP^T (legs: dstape 0 / 1, ms per backward).

    python tools/tape_ablation.py [--quick] [--dstape-only]
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_pldi_tangzwjzyz22_b200 as ft  # noqa: E402

# (name, B, H, L, d, w, dil): a (d, w) grid for the tensor-core family (w <= 64) and the C2 shapes
TC_CASES = [(f"d{d}_w{w}", 1, max(1, 16 * 64 // d), 8192, d, w, 1)
            for d in (64, 128, 256, 512) for w in (8, 32, 64)] + [("C2a", 1, 8, 10000, 512, 32, 1)]
SIMT_CASES = [("C2a", 1, 8, 10000, 512, 32, 1), ("C2b", 1, 12, 4096, 64, 256, 1), ("d64_w32", 1, 16, 8192, 64, 32, 1)]
FLUSH = None


def timed(fn, n=20, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    tot = 0.0
    for _ in range(n):
        FLUSH.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        b.synchronize()
        tot += a.elapsed_time(b)
    return tot / n


def run(name, B, H, L, d, w, dil, dt, knobs):
    dev = torch.device("cuda:0")
    q, k, v, g = [(torch.rand(B, H, L, d, device=dev) * 2 - 1).to(dt) for _ in range(4)]
    res = {"case": name, "dtype": "f32" if dt == torch.float32 else "bf16", "shape": [B, H, L, d, w, dil],
           "family": "simt" if knobs.get("path") == "simt" else "tensor cores (band kernels)",
           "tape_extra_bytes_per_step": 3 * ft.tape_bytes(q, w)}

    def rec():
        out, lse = ft.fwd(q, k, v, w, dil)
        ft.bwd(q, k, v, out, lse, g, w, dil)

    def tap():
        out, lse, tape = ft.fwd_tape(q, k, v, w, dil)
        ft.bwd_tape(q, k, v, out, lse, tape, g, w, dil)

    with ft.knobs(**knobs):
        res["recompute_ms"] = timed(rec)
        res["tape_ms"] = timed(tap)
    res["tape_speedup"] = res["recompute_ms"] / res["tape_ms"]
    print(json.dumps(res), flush=True)


DS_CASES = [(f"d{d}_w{w}", 1, max(1, 16 * 64 // d), 8192, d, w, 1)
            for d in (64, 128, 256, 512) for w in (8, 16, 32)] + [("C2a", 8, 1, 10000, 512, 32, 1),
                                                               ("C5_w32", 64, 1, 32768, 64, 32, 1)]


def run_ds(name, B, H, L, d, w, dil, dt=torch.float32):
    dev = torch.device("cuda:0")
    q, k, v, g = [(torch.rand(B, H, L, d, device=dev) * 2 - 1).to(dt) for _ in range(4)]
    out, lse = ft.fwd(q, k, v, w, dil)
    res = {"case": name, "dtype": "f32" if dt == torch.float32 else "bf16", "shape": [B, H, L, d, w, dil],
           "family": "dS tape (tensor cores)",
           "tape_bytes_per_row": 2 * 4 * ((2 * min(w, L) + 4 + 3) // 4 * 4)}
    for leg in (0, 1):
        # leg 1 forces the tape (knob value 2) below the library's d >= 256 threshold too
        with ft.knobs(dstape=2 * leg):
            res[["recompute_bwd_ms", "dstape_bwd_ms"][leg]] = timed(lambda: ft.bwd(q, k, v, out, lse, g, w, dil))
    res["dstape_speedup"] = res["recompute_bwd_ms"] / res["dstape_bwd_ms"]
    print(json.dumps(res), flush=True)


def main():
    global FLUSH
    ap = argparse.ArgumentParser()
    ap.add_argument("--quick", action="store_true")
    ap.add_argument("--dstape-only", action="store_true")
    a = ap.parse_args()
    FLUSH = torch.empty(256 << 20, dtype=torch.uint8, device="cuda:0")
    for dt in (torch.float32, torch.bfloat16):
        for c in DS_CASES:
            if dt == torch.bfloat16 and c[4] == 64 and c[5] <= 32:
                continue   # d = 64, w <= 32 runs on the narrow kernels (no tape)
            run_ds(*c, dt=dt)
    if a.dstape_only:
        return
    for c in TC_CASES[-4:] if a.quick else TC_CASES:
        run(*c, torch.bfloat16, {"narrow": 0})
    for c in SIMT_CASES[:1] if a.quick else SIMT_CASES:
        run(*c, torch.float32, {"path": "simt"})


if __name__ == "__main__":
    main()
