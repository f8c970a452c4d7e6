"""A/B step timing with no per-launch events (those sit between launches and break
programmatic dependent launch).  Runs each env setting in a subprocess.
Usage: python tools/step_ab.py [workload] VAR=a,b [VAR2=c,d ...]
"""
import itertools
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CHILD = r"""
import sys, torch
sys.path.insert(0, %r)
import bench, paper_conf_pldi_tangzwjzyz22_b200 as ft
WL = bench.WORKLOADS[%r]
B, H, L, d, w, dil = WL[:6]
hd = WL[7] if len(WL) > 7 else None
dev = torch.device("cuda:0")
g = torch.Generator(device=dev).manual_seed(0)
q, k, v, dout = (torch.randn(B, H, L, d, device=dev, dtype=torch.bfloat16, generator=g) for _ in range(4))
out, lse = ft.fwd(q, k, v, w, dil, dilated_heads=hd)
dq, dk, dv = (torch.empty_like(q) for _ in range(3))
ws = torch.empty(max(ft.workspace_bytes(q, w, dil), 16), dtype=torch.uint8, device=dev)
flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
ts = []
for i in range(60):
    flush.zero_()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    ft.fwd(q, k, v, w, dil, out=out, lse=lse, dilated_heads=hd)
    ft.bwd(q, k, v, out, lse, dout, w, dil, dq=dq, dk=dk, dv=dv, workspace=ws, dilated_heads=hd)
    b.record()
    torch.cuda.synchronize()
    if i >= 10:
        ts.append(a.elapsed_time(b))
ts.sort()
print(ts[len(ts) // 2], sum(ts) / len(ts))
"""


def main():
    wl = "C2a"
    args = sys.argv[1:]
    if args and "=" not in args[0]:
        wl = args.pop(0)
    axes = [(a.split("=")[0], a.split("=")[1].split(",")) for a in args]
    for rep in range(2):
        for combo in itertools.product(*[vals for _, vals in axes]):
            env = dict(os.environ)
            tag = []
            for (name, _), val in zip(axes, combo):
                env[name] = val
                tag.append(f"{name}={val}")
            r = subprocess.run([sys.executable, "-c", CHILD % (ROOT, wl)], env=env, capture_output=True,
                               text=True)
            if r.returncode:
                print(" ".join(tag), "FAILED", r.stderr[-500:])
                continue
            med, mean = map(float, r.stdout.split())
            print(json.dumps({"workload": wl, "env": " ".join(tag), "median_ms": round(med, 4),
                              "mean_ms": round(mean, 4)}))


if __name__ == "__main__":
    main()
