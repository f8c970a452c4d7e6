"""fwd / bwd time of one workload against a debug knob's values (A/B probe, bit-identity checked).
Usage: python tools/knob_probe.py KNOB v1,v2,... [--workload C2a] [--dtype f32,bf16] [--L L]"""
import argparse
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_pldi_tangzwjzyz22_b200 as ft  # noqa: E402

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


ap = argparse.ArgumentParser()
ap.add_argument("knob")
ap.add_argument("values")
ap.add_argument("--workload", default="C2a")
ap.add_argument("--dtype", default="f32,bf16")
ap.add_argument("--L", type=int, default=0)
ap.add_argument("--knob2", default="")
ap.add_argument("--rounds", type=int, default=4)
a = ap.parse_args()
B, H, L, d, w, dil = bench.WORKLOADS[a.workload][:6]
if a.L:
    L = a.L
extra = [kv.split("=") for kv in a.knob2.split(",") if kv]
for k2, v2 in extra:
    ft.debug_set(k2, int(v2))
for dn in a.dtype.split(","):
    dt = torch.float32 if dn == "f32" else torch.bfloat16
    g = torch.Generator(device=dev).manual_seed(0)
    q, k, v, dout = (torch.rand(B, H, L, d, device=dev, generator=g).mul_(2).sub_(1).to(dt) for _ in range(4))
    out, lse = ft.fwd(q, k, v, w, dil)
    dq, dk, dv = (torch.empty_like(q) for _ in range(3))
    ws = torch.empty(max(ft.workspace_bytes(q, w, dil), 16), dtype=torch.uint8, device=dev)
    ref = None
    old = ft.debug_get(a.knob)
    vals = [int(x) for x in a.values.split(",")]
    best = {}
    same = {}
    for rnd in range(a.rounds):   # interleaved rounds; the minimum of the per-round medians
        for val in vals:
            ft.debug_set(a.knob, val)
            tf = timeit(lambda: ft.fwd(q, k, v, w, dil, out=out, lse=lse))
            tb = timeit(lambda: ft.bwd(q, k, v, out, lse, dout, w, dil, dq=dq, dk=dk, dv=dv, workspace=ws))
            ts = timeit(lambda: (ft.fwd(q, k, v, w, dil, out=out, lse=lse),
                                 ft.bwd(q, k, v, out, lse, dout, w, dil, dq=dq, dk=dk, dv=dv, workspace=ws)))
            got = torch.cat([out.flatten(), lse.flatten().to(dt), dq.flatten(), dk.flatten(), dv.flatten()])
            if ref is None:
                ref = got.clone()
            same[val] = same.get(val, True) and torch.equal(got, ref)
            b = best.get(val, (1e9, 1e9, 1e9))
            best[val] = (min(b[0], tf), min(b[1], tb), min(b[2], ts))
    for val in vals:
        tf, tb, ts = best[val]
        print(f"{a.workload} {dn:5s} L={L} {a.knob}={val:5d} fwd={tf * 1e3:7.1f}us bwd={tb * 1e3:7.1f}us "
              f"step={ts * 1e3:7.1f}us  {'bit-identical to the first' if same[val] else 'DIFFERENT'}", flush=True)
    ft.debug_set(a.knob, old)
