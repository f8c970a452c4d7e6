"""Phase timeline of the tensor-core kernels from ft_winattn_debug_trace (profiling aid).

    python tools/trace_phases.py [--workload C2a]

Prints, per kernel mode, the median over CTAs/tiles of each pipeline phase in thousands of
SM cycles (kclk; the kernels stamp clock64, so only differences within a CTA are meaningful).
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

EV = ["prod_g1_start", "prod_out_end", "mma_g1_ready", "mma_s_commit", "mma_p_seen",
      "mma_out_end", "sm_s_seen", "sm_p_arrive", "epi_first", "epi_done"]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--workload", default="C2a")
    a = ap.parse_args()
    B, H, L, d, w, dil, _ = bench.WORKLOADS[a.workload]
    lib = ft.load_library()
    lib.ft_winattn_debug_trace.argtypes = [ctypes.c_int, ctypes.c_void_p]
    dev = torch.device("cuda:0")
    x = [(torch.rand(B, H, L, d, device=dev) * 2 - 1).to(torch.bfloat16) for _ in range(4)]
    q, k, v, g = x
    out, lse = ft.fwd(q, k, v, w, dil)
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    bufs = [torch.zeros(148 * 8 * 48, dtype=torch.int64, device=dev) for _ in range(3)]
    for m in range(3):
        lib.ft_winattn_debug_trace(m, bufs[m].data_ptr())
    out, lse = ft.fwd(q, k, v, w, dil)
    ft.bwd(q, k, v, out, lse, g, w, dil)
    torch.cuda.synchronize()
    for m in range(3):
        lib.ft_winattn_debug_trace(m, None)
    for m, name in enumerate(["FWD", "BWDQ", "BWDKV"]):
        t = bufs[m].view(148, 8, 48).cpu().double()
        valid = (t[:, :, :10] > 0).all(dim=2) & (t[:, :, 12] > 0) & (t[:, :, 13] > 0)
        t0 = t[:, 0:1, 0:1]
        t = (t - t0) / 1e3
        print(f"== {name}: tiles traced {int(valid.sum())} (kclk)")
        def med(x):
            return float(x[valid].median())
        print(f"  GEMM1 (mma ready -> s commit)     {med(t[:,:,3]-t[:,:,2]):7.2f} kclk")
        print(f"  s commit -> softmax start         {med(t[:,:,6]-t[:,:,3]):7.2f}")
        print(f"  softmax (s seen -> p arrive)      {med(t[:,:,7]-t[:,:,6]):7.2f}")
        if name == "FWD":
            print(f"    pass 1 (max)                    {med(t[:,:,10]-t[:,:,6]):7.2f}")
            print(f"    wait P buffer free              {med(t[:,:,11]-t[:,:,10]):7.2f}")
            print(f"    pass 2 (exp, P -> smem)         {med(t[:,:,7]-t[:,:,11]):7.2f}")
        if name == "BWDKV" and float(t[:, :, 11].max()) > 0:   # dS tape: build phases
            print(f"    xt: loop top -> A operands free {med(t[:,:,10]-t[:,:,6]):7.2f}")
            print(f"    xt: -> first tape slot landed   {med(t[:,:,11]-t[:,:,10]):7.2f}")
            print(f"    xt: -> last tape slot landed    {med(t[:,:,15]-t[:,:,11]):7.2f}")
            print(f"    xt: -> p arrive (build)         {med(t[:,:,7]-t[:,:,15]):7.2f}")
        print(f"  p arrive -> mma sees p            {med(t[:,:,4]-t[:,:,7]):7.2f}")
        print(f"  output MMAs issued (p -> out end) {med(t[:,:,5]-t[:,:,4]):7.2f}")
        print(f"    p seen -> o_empty passed        {med(t[:,:,12]-t[:,:,4]):7.2f}")
        print(f"    o_empty -> first O block full   {med(t[:,:,13]-t[:,:,12]):7.2f}")
        if name == "FWD":
            print(f"    p seen -> G(j+1) issued         {med(t[:,:,14]-t[:,:,4]):7.2f}")
        print(f"  epilogue (first o_full -> done)   {med(t[:,:,9]-t[:,:,8]):7.2f}")
        print(f"  tile period (g1 ready j -> j+1)   {float((t[:,1:,2]-t[:,:-1,2])[valid[:,1:] & valid[:,:-1]].median()):7.2f}")
        print(f"  producer span per tile            {med(t[:,:,1]-t[:,:,0]):7.2f}")
        print(f"  first tile start (median over CTAs) {float(t[:,0,2][valid[:,0]].median()):7.2f}")



if __name__ == "__main__":
    main()
