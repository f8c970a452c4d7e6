"""BASELINE configs[4] sweep on one B200: H in {8, 16, 32, 64} x L in {4096, 8192, 16384, 32768},
d = 64, w in {32, 256}, bf16 fwd+bwd.  Per point: ms per step (CUDA events,
mean of N after 3 warm-ups; 252 MiB L2 flush between steps when the inputs fit in L2), tokens/s,
head-tokens/s, the kernel family the dispatcher chose, and the step's fraction of the §8(d) HBM
roofline (fwd 4de+4 + bwd 8de+4 bytes per row against the measured peak).

    python tools/sweep_c5.py [--steps 20]
"""
import argparse
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_pldi_tangzwjzyz22_b200 as ft  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--steps", type=int, default=20)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    peak = bench.load_peaks()[0]
    flush = torch.empty(2 * bench.L2_BYTES, dtype=torch.uint8, device=dev)
    for w in (32, 256):
        for H in (8, 16, 32, 64):
            for L in (4096, 8192, 16384, 32768):
                d, e = 64, 2
                q, k, v, g = [(torch.rand(1, H, L, d, device=dev) * 2 - 1).to(torch.bfloat16) for _ in range(4)]
                ws = torch.empty(max(ft.workspace_bytes(q, w, 1), 16), dtype=torch.uint8, device=dev)
                small = 4 * q.numel() * e <= bench.L2_BYTES
                out, lse = ft.fwd(q, k, v, w)
                dq, dk, dv = (torch.empty_like(q) for _ in range(3))

                def step():
                    ft.fwd(q, k, v, w, out=out, lse=lse)
                    ft.bwd(q, k, v, out, lse, g, w, dq=dq, dk=dk, dv=dv, workspace=ws)

                for _ in range(3):
                    step()
                torch.cuda.synchronize()
                tot = 0.0
                for _ in range(a.steps):
                    if small:
                        flush.zero_()
                    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    s0.record()
                    step()
                    s1.record()
                    torch.cuda.synchronize()
                    tot += s0.elapsed_time(s1)
                ms = tot / a.steps
                pf, nf = ft.plan(False, 1, H, L, d, w, 1, ft.FT_BF16)
                pb, nb = ft.plan(True, 1, H, L, d, w, 1, ft.FT_BF16)
                alg = bench.step_bytes_per_row(d, e) * H * L
                print(json.dumps({"H": H, "L": L, "d": d, "w": w, "ms_per_step": round(ms, 4),
                                  "tokens_per_s": L / (ms / 1e3), "head_tokens_per_s": H * L / (ms / 1e3),
                                  "bwd_launches": nb, "hbm_step_frac": alg / (ms / 1e3) / 1e9 / peak,
                                  "l2_flushed": small}), flush=True)
                del q, k, v, g, out, lse, dq, dk, dv, ws
                torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
