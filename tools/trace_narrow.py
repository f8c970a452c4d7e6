"""Phase timeline of the narrow (d = 64, w <= 32) backward kernels (profiling aid).

    python tools/trace_narrow.py [--workload C5_w32]

Uses ft_winattn_debug_trace (modes 1 = NQ, 2 = NKV); prints, per event of
tc_narrow_bwd.cu's trace_ev list, the median over CTAs and traced tiles 1..7 of its time
relative to the tile's MMA iteration start (SM cycles), and the median tile period.
"""
import argparse
import ctypes
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_pldi_tangzwjzyz22_b200 as ft  # noqa: E402

EV = ["mma iter start", "S(j) issued", "out(j-1) issued", "dP(j) issued", "sm s_full seen",
      "sm S/dP loaded", "sm operand buf free", "sm pair barrier", "sm p_done", "sm acc seen",
      "sm drained", "prod loads issued", "halo converted", "mma sees s_full", "conv sees s_full", "sm setup done", "sm acc loaded", "conv table published"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C5_w32")
    ap.add_argument("--raw", action="store_true")
    ap.add_argument("--raw-ctas", type=int, nargs="*", default=[0, 77])
    a = ap.parse_args()
    B, H, L, d, w, dil, _ = bench.WORKLOADS[a.workload]
    lib = ft.load_library()
    lib.ft_winattn_debug_trace.argtypes = [ctypes.c_int, ctypes.c_void_p]
    dev = torch.device("cuda:0")
    q, k, v, g = [(torch.rand(B, H, L, d, device=dev) * 2 - 1).to(torch.bfloat16) for _ in range(4)]
    out, lse = ft.fwd(q, k, v, w, dil)
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    bufs = {m: torch.zeros(148 * 8 * 48, dtype=torch.int64, device=dev) for m in (1, 2)}
    for m, b in bufs.items():
        lib.ft_winattn_debug_trace(m, b.data_ptr())
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    for m in bufs:
        lib.ft_winattn_debug_trace(m, None)
    for m, name in ((1, "NQ"), (2, "NKV")):
        t = bufs[m].view(148, 8, 48).cpu().double()
        base = t[:, :, 0:1]
        rel = t[:, 1:, :len(EV)] - base[:, 1:]
        ok = (t[:, 1:, :len(EV)] > 0).all(dim=2)
        print(f"== {name}")
        for e, nm in enumerate(EV):
            print(f"  {nm:22s} {float(rel[:, :, e][ok].median()):7.0f} clk")
        if a.raw:
            for c in a.raw_ctas:
                t0 = t[c, 1, 0]
                print(f"  CTA {c} raw (clk from tile 1 start):")
                for jj in range(1, 8):
                    print("   tile", jj, " ".join(f"{int(t[c, jj, e] - t0):6d}" for e in range(len(EV))))
        per = t[:, 2:, 0] - t[:, 1:-1, 0]
        print(f"  tile period            {float(per[(t[:, 2:, 0] > 0) & (t[:, 1:-1, 0] > 0)].median()):7.0f} clk")


if __name__ == "__main__":
    main()
