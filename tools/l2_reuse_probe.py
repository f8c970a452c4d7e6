"""Probe: how fast is the d = 512 BWDKV kernel when its inputs are L2-resident?

In one ft_winattn_bwd call BWDQ reads q, k, v, dout and BWDKV reads them again. At C2a's size
(4 x 82 MB) the second read comes from HBM; at a size whose four inputs fit in L2 it comes
from L2. Comparing the per-tile time of the two says whether running the backward in L2-sized
row groups (BWDQ then BWDKV per group) would pay. L2 is flushed before every call.
Usage: python tools/l2_reuse_probe.py
"""
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_pldi_tangzwjzyz22_b200 as ft  # noqa: E402


def run(B, H, L, d=512, w=32, reps=20):
    dev = torch.device("cuda:0")
    g = torch.Generator(device=dev).manual_seed(0)
    q, k, v, dout = (torch.randn(B, H, L, d, device=dev, dtype=torch.bfloat16, generator=g) for _ in range(4))
    out, lse = ft.fwd(q, k, v, w)
    dq, dk, dv = (torch.empty_like(q) for _ in range(3))
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    ev = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
    t = {"q": [], "kv": []}
    for i in range(reps + 3):
        flush.zero_()
        s0, e = ev(), [ev(), ev()]
        s0.record()
        with ft.profile_events(e):
            ft.bwd(q, k, v, out, lse, dout, w, dq=dq, dk=dk, dv=dv)
        torch.cuda.synchronize()
        if i >= 3:
            t["q"].append(s0.elapsed_time(e[0]))
            t["kv"].append(e[0].elapsed_time(e[1]))
    tiles = B * H * ((L + 127) // 128)
    mq, mkv = (sorted(x)[len(x) // 2] for x in (t["q"], t["kv"]))
    waves = tiles / 148
    print(f"B={B} H={H} L={L}: tiles {tiles} ({waves:.2f} per SM)  inputs {4 * B * H * L * d * 2 / 1e6:.0f} MB  "
          f"BWDQ {mq * 1e3:.1f} us  BWDKV {mkv * 1e3:.1f} us  "
          f"per tile-wave: BWDQ {mq * 1e3 / max(waves, 1):.1f} BWDKV {mkv * 1e3 / max(waves, 1):.1f} us")


if __name__ == "__main__":
    for B, H, L in [(1, 1, 18944), (1, 2, 18944), (1, 3, 18944), (1, 8, 10000), (1, 16, 18944)]:
        run(B, H, L)
