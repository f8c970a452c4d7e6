"""Phase breakdown of the wide-window backward kernels (csrc/tc_wide_bwd.cu) from
ft_winattn_debug_trace, modes 1 (dQ kernel) and 2 (dK/dV kernel).  Profiling aid.

    python tools/trace_wide_bwd.py [--workload C5_w256]
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


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C5_w256")
    a = ap.parse_args()
    B, H, L, d, w, dil, _ = bench.WORKLOADS[a.workload]
    lib = ft.load_library()
    lib.ft_winattn_debug_trace.argtypes = [ctypes.c_int, ctypes.c_void_p]
    dev = torch.device("cuda:0")
    q, k, v, g = [(torch.rand(B, H, L, d, device=dev) * 2 - 1).to(torch.bfloat16) for _ in range(4)]
    out, lse = ft.fwd(q, k, v, w, dil)
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    bufs = [torch.zeros(148 * 8 * 48, dtype=torch.int64, device=dev) for _ in range(2)]
    for m in (1, 2):
        lib.ft_winattn_debug_trace(m, bufs[m - 1].data_ptr())
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    for m in (1, 2):
        lib.ft_winattn_debug_trace(m, None)
    for name, buf in (("dQ kernel", bufs[0]), ("dK/dV kernel", bufs[1])):
        t = buf.view(148, 8, 48).cpu().double()
        sel = t[:, 1:7, :]
        ok = (sel[:, :, 0] > 0) & (sel[:, :, 6] > 0)
        med = lambda x: float(x[ok].median()) / 1e3  # noqa: E731
        period = t[:, 2:8, 0] - t[:, 1:7, 0]
        pok = (t[:, 2:8, 0] > 0) & (t[:, 1:7, 0] > 0)
        print(f"== {a.workload} {name}: tile period {float(period[pok].median()) / 1e3:.2f} us")
        for label, s in [("softmax S/dP wait", 1), ("softmax compute", 2), ("issuer A region wait", 10),
                         ("issuer A ring wait", 11), ("issuer B region wait", 14), ("issuer B ring wait", 15),
                         ("issuer C p_full wait", 20), ("issuer C o_empty wait", 21)]:
            print(f"  {label:28s} {med(sel[:, :, s]):7.2f}")
        print(f"  {'epilogue (o_full -> done)':28s} {med(sel[:, :, 31] - sel[:, :, 30]):7.2f}")


if __name__ == "__main__":
    main()
