"""Tape vs recompute on B200 (Fig. 18): the paper's
selective materialization decides per intermediate whether the gradient program reads it from a
tape or recomputes it.  Here the intermediate is the band score s_ij = q_i . k_j:

  recompute : ft_winattn_fwd + ft_winattn_bwd (saves lse only; bwd recomputes q_i . k_j)
  tape      : ft_winattn_fwd_tape + ft_winattn_bwd_tape (fwd writes s, fp32 [rows][2w+1]; bwd reads it)

both on the CUDA-core kernels (FT_WINATTN_PATH=simt), plus the tensor-core recompute path for
bf16.  Prints ms per fwd+bwd step (CUDA events, mean of 10 after 3 warm-ups) and the tape's
extra HBM bytes per step (write + read).

    python tools/tape_ablation.py
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_pldi_tangzwjzyz22_b200 as ft  # noqa: E402

CASES = [  # (name, B, H, L, d, w, dil)
    ("C2a", 1, 8, 10000, 512, 32, 1),
    ("C2b", 1, 12, 4096, 64, 256, 1),
    ("d64_w32", 1, 16, 8192, 64, 32, 1),
    ("d128_w64", 1, 8, 8192, 128, 64, 1),
]


def timed(fn, n=10, warm=3):
    for _ in range(warm):
        fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n):
        fn()
    b.record()
    torch.cuda.synchronize()
    return a.elapsed_time(b) / n


def main():
    dev = torch.device("cuda:0")
    for name, B, H, L, d, w, dil in CASES:
        for dt in (torch.float32, torch.bfloat16):
            q, k, v, g = [(torch.rand(B, H, L, d, device=dev) * 2 - 1).to(dt) for _ in range(4)]
            res = {"case": name, "dtype": "f32" if dt == torch.float32 else "bf16",
                   "shape": [B, H, L, d, w, dil],
                   "tape_extra_bytes_per_step": 2 * ft.tape_bytes(q, w)}

            def rec():
                out, lse = ft.fwd(q, k, v, w, dil)
                ft.bwd(q, k, v, out, lse, g, w, dil)

            def tap():
                out, lse, tape = ft.fwd_tape(q, k, v, w, dil)
                ft.bwd_tape(q, k, v, out, lse, tape, g, w, dil)

            os.environ["FT_WINATTN_PATH"] = "simt"
            res["simt_recompute_ms"] = timed(rec)
            res["simt_tape_ms"] = timed(tap)
            os.environ.pop("FT_WINATTN_PATH")
            if dt == torch.bfloat16:
                res["tc_recompute_ms"] = timed(rec)
            print(json.dumps(res), flush=True)
            del q, k, v, g
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
