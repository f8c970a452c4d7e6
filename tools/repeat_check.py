"""Repeatability sweep: every tensor-core family's fwd + bwd run N times on one input, every output
compared bit for bit with the first run (the kernels own their output rows, no atomics, so any
difference is a race).  Alternates the PDL knob.  Usage: python tools/repeat_check.py [N]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_tangzwjzyz22_b200 as ft  # noqa: E402
from synth import WinAttnShape, make_inputs  # noqa: E402

CASES = [("narrow bf16 d64 w32", (1, 16, 8192, 64, 32, 1), "bf16"),
         ("band bf16 d512 w32 (C2a)", (1, 8, 10000, 512, 32, 1), "bf16"),
         ("band32 fp32 d512 w32 (C2a)", (1, 8, 10000, 512, 32, 1), "f32"),
         ("band32 fp32 d64 w32", (1, 16, 8192, 64, 32, 1), "f32"),
         ("wide bf16 d64 w256 d2", (1, 12, 16384, 64, 256, 2), "bf16"),
         ("wide bf16 d128 w256", (1, 12, 4096, 128, 256, 1), "bf16"),
         ("band32 WIDE fp32 d64 w256", (1, 12, 4096, 64, 256, 1), "f32"),
         ("band32 WIDE fp32 d128 w100", (1, 8, 4096, 128, 100, 1), "f32"),
         ("band bf16 d256 w16 d3", (1, 4, 6000, 256, 16, 3), "bf16"),
         ("narrow bf16 d64 w20 d3", (2, 6, 5001, 64, 20, 3), "bf16"),
         ("wide bf16 d64 w100 d4", (1, 6, 9001, 64, 100, 4), "bf16"),
         ("wide bf16 d128 w130 d2", (1, 4, 6001, 128, 130, 2), "bf16"),
         ("band32 fp32 d256 w32 d5 (tape)", (1, 3, 7001, 256, 32, 5), "f32"),
         ("band32 WIDE fp32 d64 w300 d3", (1, 4, 7001, 64, 300, 3), "f32"),
         ("very wide bf16 d64 w2000 (chunk)", (1, 2, 5000, 64, 2000, 1), "bf16")]


def main():
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 50
    dev = torch.device("cuda:0")
    total_bad = 0
    for name, shape, dt in CASES:
        sh = WinAttnShape(*shape)
        x = make_inputs(sh, 31, dt)
        q, k, v, g = (x[t].to(dev) for t in ("q", "k", "v", "dout"))
        ref, bad = None, 0
        for it in range(n):
            with ft.knobs(pdl=1 if it % 3 else 0):
                out, lse = ft.fwd(q, k, v, sh.w, sh.dilation)
                r = (out, lse) + ft.bwd(q, k, v, out, lse, g, sh.w, sh.dilation)
            torch.cuda.synchronize()
            if ref is None:
                ref = [t.clone() for t in r]
                continue
            if not all(torch.equal(a, b) for a, b in zip(r, ref)):
                bad += 1
        total_bad += bad
        print(f"{name:32s} {shape}: {bad} of {n - 1} repeats differ", flush=True)
    # one-call fwd + bwd (lse hand-off), per-head dilation (two streams), score tape
    extra = [("fwd_bwd bf16 d512", (1, 8, 10000, 512, 32, 1), "bf16", "fwd_bwd"),
             ("fwd_bwd fp32 d512", (1, 8, 10000, 512, 32, 1), "f32", "fwd_bwd"),
             ("fwd_bwd narrow bf16", (1, 16, 8192, 64, 32, 1), "bf16", "fwd_bwd"),
             ("mixed dilation bf16 d512", (1, 8, 10000, 512, 32, 4), "bf16", "mixed"),
             ("mixed dilation fp32 d512", (1, 8, 10000, 512, 32, 4), "f32", "mixed"),
             ("score tape bf16 d64", (1, 8, 4096, 64, 20, 1), "bf16", "tape")]
    for name, shape, dt, kind in extra:
        sh = WinAttnShape(*shape)
        x = make_inputs(sh, 32, dt)
        q, k, v, g = (x[t].to(dev) for t in ("q", "k", "v", "dout"))
        ref, bad = None, 0
        for it in range(n):
            if kind == "fwd_bwd":
                r = ft.fwd_bwd(q, k, v, g, sh.w, sh.dilation)
            elif kind == "mixed":
                out, lse = ft.fwd(q, k, v, sh.w, sh.dilation, dilated_heads=2)
                r = (out, lse) + ft.bwd(q, k, v, out, lse, g, sh.w, sh.dilation, dilated_heads=2)
            else:
                out, lse, tp = ft.fwd_tape(q, k, v, sh.w, sh.dilation)
                r = (out, lse) + ft.bwd_tape(q, k, v, out, lse, tp, g, sh.w, sh.dilation)
            torch.cuda.synchronize()
            if ref is None:
                ref = [t.clone() for t in r]
                continue
            if not all(torch.equal(a, b) for a, b in zip(r, ref)):
                bad += 1
        total_bad += bad
        print(f"{name:32s} {shape}: {bad} of {n - 1} repeats differ", flush=True)
    print("total differing repeats:", total_bad)


if __name__ == "__main__":
    main()
