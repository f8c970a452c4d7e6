"""Slot / tile timeline of the fp32 tensor-core kernels (csrc/tc_band32.cu) from
ft_winattn_debug_trace (profiling aid).

    python tools/trace32.py [--workload C2a]

For CTA 0 of each kernel mode it prints, per ring slot in walk order, the clock64 stamps (kclk
from the first producer issue) of: producer TMA issue, converter start / done, MMA issue start /
end -- and per tile the softmax and epilogue events; then the medians over all CTAs of the
per-slot gaps (TMA issue -> converter start = load latency, converter time, converter done ->
MMA start, MMA issue time)."""
import argparse
import ctypes
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_pldi_tangzwjzyz22_b200 as ft  # noqa: E402

TR_SLOTS, TR_TILES = 96, 4
PER = TR_SLOTS * 5 + TR_TILES * 16


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C2a")
    ap.add_argument("--slots", type=int, default=40)
    a = ap.parse_args()
    B, H, L, d, w, dil, _ = bench.WORKLOADS[a.workload][:7]
    lib = ft.load_library()
    lib.ft_winattn_debug_trace.argtypes = [ctypes.c_int, ctypes.c_void_p]
    dev = torch.device("cuda:0")
    q, k, v, g = [torch.rand(B, H, L, d, device=dev) * 2 - 1 for _ in range(4)]
    out, lse = ft.fwd(q, k, v, w, dil)
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    bufs = [torch.zeros(148 * PER, dtype=torch.int64, device=dev) for _ in range(3)]
    for m in range(3):
        lib.ft_winattn_debug_trace(m, bufs[m].data_ptr())
    out, lse = ft.fwd(q, k, v, w, dil)
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    for m in range(3):
        lib.ft_winattn_debug_trace(m, None)
    for m, name in enumerate(["FWD", "BWDQ", "BWDKV"]):
        t = bufs[m].view(148, PER).cpu().double()
        s = t[:, :TR_SLOTS * 5].view(148, TR_SLOTS, 5)
        tl = t[:, TR_SLOTS * 5:].view(148, TR_TILES, 16)
        t0 = s[:, 0:1, 0:1]
        s = (s - t0) / 1e3
        tl = (tl - t0[:, :, :1]) / 1e3
        print(f"== {name} (CTA 0, kclk)   prod  cv0  cv1  mma0 mma1")
        for i in range(min(a.slots, TR_SLOTS)):
            r = s[0, i]
            if int(bufs[m].view(148, PER)[0, i * 5]) == 0:
                break
            r = torch.where(bufs[m].view(148, PER)[0, i * 5:(i + 1) * 5].cpu() == 0, torch.full_like(r, float("nan")), r)
            print(f"  slot {i:3d} " + " ".join(f"{x:6.1f}" for x in r.tolist()))
        for j in range(TR_TILES):
            print(f"  tile {j}: " + " ".join("   -   " if x < -1e6 else f"{x:7.1f}" for x in tl[0, j].tolist()))
        ok = (bufs[m].view(148, PER)[:, :TR_SLOTS * 5].view(148, TR_SLOTS, 5) > 0).all(dim=2).cpu()
        def med(x):
            return float(x[ok].median()) if ok.any() else float("nan")
        print(f"  medians over slots: tma->conv {med(s[:, :, 1] - s[:, :, 0]):.2f}  conv {med(s[:, :, 2] - s[:, :, 1]):.2f}"
              f"  conv->mma {med(s[:, :, 3] - s[:, :, 2]):.2f}  mma issue {med(s[:, :, 4] - s[:, :, 3]):.2f}"
              f"  slot period {float((s[:, 1:, 4] - s[:, :-1, 4])[ok[:, 1:] & ok[:, :-1]].median()):.2f} kclk")


if __name__ == "__main__":
    main()
