"""Phase timeline of the fused d = 64, w <= 32 backward (csrc/tc_narrow_fused.cu; profiling aid).

    python tools/trace_fused.py [--workload C5_w32] [--raw]

Uses ft_winattn_debug_trace mode 1; prints, per trace_ev event, the median over CTAs and traced
items 9..15 of its time relative to the item's MMA-issuer iteration start (SM cycles), and the
median item period.
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

EV = ["mma iter start", "S(j) issued", "out(j) issued", "dP(j) issued", "sm s_full seen",
      "sm dp_full seen", "sm p_done", "sm drain(j-1) done", "prod QO(j) issued", "prod K(j) issued",
      "prod V(j) issued", "conv s_full seen", "out A mmas issued", "conv done", "out accfree ok",
      "out(j) conv ok", "mma s_free seen", "sm pair barrier", "out(j) p_done ok", "out dqfree ok",
      "out mmas issued", "sm drain(j-1) dq ld", "sm drain(j-1) X ld", "i1 vfull ok", "i1 dP mmas issued",
      "i1 dp_free(j-1) ok", "i1 conv(j) ok"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C5_w32")
    ap.add_argument("--raw", action="store_true")
    a = ap.parse_args()
    B, H, L, d, w, dil, _ = bench.WORKLOADS[a.workload]
    lib = ft.load_library()
    lib.ft_winattn_debug_trace.argtypes = [ctypes.c_int, ctypes.c_void_p]
    dev = torch.device("cuda:0")
    q, k, v, g = [(torch.rand(B, H, L, d, device=dev) * 2 - 1).to(torch.bfloat16) for _ in range(4)]
    out, lse = ft.fwd(q, k, v, w, dil)
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    buf = torch.zeros(148 * 8 * 48, dtype=torch.int64, device=dev)
    lib.ft_winattn_debug_trace(1, buf.data_ptr())
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    lib.ft_winattn_debug_trace(1, None)
    n = len(EV)
    t = buf.view(148, 8, 48).cpu().double()
    base = t[:, :, 0:1]
    rel = t[:, 1:, :n] - base[:, 1:]
    for e, nm in enumerate(EV):
        ok = (t[:, 1:, e] > 0) & (t[:, 1:, 0] > 0)
        if ok.any():
            print(f"  {e:2d} {nm:22s} {float(rel[:, :, e][ok].median()):7.0f} clk")
    per = t[:, 2:, 0] - t[:, 1:-1, 0]
    print(f"  item period             {float(per[(t[:, 2:, 0] > 0) & (t[:, 1:-1, 0] > 0)].median()):7.0f} clk")
    if a.raw:
        for c in (0, 77):
            t0 = t[c, 1, 0]
            print(f"  CTA {c} raw (clk from item 9 start):")
            for jj in range(1, 8):
                print("   item", jj + 8, " ".join(f"{int(t[c, jj, e] - t0):6d}" for e in range(n)))


if __name__ == "__main__":
    main()
