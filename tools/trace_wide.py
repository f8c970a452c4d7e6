"""Phase breakdown of the wide-window forward kernel (csrc/tc_wide.cu) from
ft_winattn_debug_trace, mode 0 (profiling aid).

    python tools/trace_wide.py [--workload C5_w256]

Prints medians over CTAs of tiles 1..6 (steady state), microseconds.
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
    q, k, v = [(torch.rand(B, H, L, d, device=dev) * 2 - 1).to(torch.bfloat16) for _ in range(3)]
    ft.fwd(q, k, v, w, dil)
    torch.cuda.synchronize()
    buf = torch.zeros(148 * 8 * 48, dtype=torch.int64, device=dev)
    lib.ft_winattn_debug_trace(0, buf.data_ptr())
    ft.fwd(q, k, v, w, dil)
    torch.cuda.synchronize()
    lib.ft_winattn_debug_trace(0, None)
    t = buf.view(148, 8, 48).cpu().double()
    sel = t[:, 1:7, :]
    ok = (sel[:, :, 0] > 0) & (sel[:, :, 6] > 0)

    def med(x):
        return float(x[ok].median()) / 1e3

    period = (t[:, 2:8, 0] - t[:, 1:7, 0])
    pok = (t[:, 2:8, 0] > 0) & (t[:, 1:7, 0] > 0)
    print(f"== {a.workload}: tile period {float(period[pok].median()) / 1e3:.2f} us")
    for name, s in [("softmax S wait", 1), ("softmax P-buffer wait", 2),
                    ("softmax compute", 3), ("  S tmem load+wait", 40), ("  exp sweep", 41),
                    ("  max exchange", 42), ("  fence + arrive", 43), ("softmax rescales (count)", 4), ("issuer A buffer-free wait", 11),
                    ("issuer A K wait", 12), ("issuer B p_full wait", 20),
                    ("issuer B o_empty wait", 21), ("issuer B V wait", 22)]:
        v = med(sel[:, :, s])
        print(f"  {name:32s} {v * 1e3 if 'count' in name else v:7.2f}")
    print(f"  {'softmax tile span':32s} {med(sel[:, :, 6] - sel[:, :, 0]):7.2f}")
    print(f"  {'epilogue (o_full seen -> done)':32s} {med(sel[:, :, 31] - sel[:, :, 30]):7.2f}")
    print(f"  {'o_full commit - softmax end':32s} {med(sel[:, :, 23] - sel[:, :, 6]):7.2f}")


if __name__ == "__main__":
    main()
