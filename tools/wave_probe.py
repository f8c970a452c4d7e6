"""Wave-quantization probe: fwd / bwd time of the d = 512 band kernels against L around
the 4-wave boundary (148 SMs, 8 units: 592 tiles at L = 9472).  Usage: python tools/wave_probe.py"""
import sys, os
import torch
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_pldi_tangzwjzyz22_b200 as ft

dev = torch.device("cuda:0")
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)


def timeit(fn, n=30):
    ts = []
    for i in range(n + 5):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize()
        if i >= 5:
            ts.append(a.elapsed_time(b))
    ts.sort()
    return ts[len(ts) // 2]


for dt in (torch.float32, torch.bfloat16):
    for L in [int(x) for x in (sys.argv[1:] or ["9472", "9473", "9600", "10000", "10112", "11000"])]:
        H, d, w = 8, 512, 32
        g = torch.Generator(device=dev).manual_seed(0)
        q, k, v, dout = (torch.rand(1, H, L, d, device=dev, generator=g).mul_(2).sub_(1).to(dt) for _ in range(4))
        out, lse = ft.fwd(q, k, v, w)
        dq, dk, dv = (torch.empty_like(q) for _ in range(3))
        ws = torch.empty(max(ft.workspace_bytes(q, w), 16), dtype=torch.uint8, device=dev)
        tf = timeit(lambda: ft.fwd(q, k, v, w, out=out, lse=lse))
        tb = timeit(lambda: ft.bwd(q, k, v, out, lse, dout, w, dq=dq, dk=dk, dv=dv, workspace=ws))
        tiles = H * ((L + 127) // 128)
        print(f"{str(dt)[6:]:8s} L={L:6d} tiles={tiles:4d} waves={tiles/148:5.2f} fwd={tf*1e3:7.1f}us "
              f"bwd={tb*1e3:7.1f}us  fwd/row={tf*1e6/(H*L):6.2f}ns bwd/row={tb*1e6/(H*L):6.2f}ns", flush=True)
