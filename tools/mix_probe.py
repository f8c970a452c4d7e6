import os, sys, torch, subprocess
sys.path.insert(0, "/root/repo")
CH = r'''
import sys, torch
sys.path.insert(0, "/root/repo")
import paper_conf_pldi_tangzwjzyz22_b200 as ft
dev = torch.device("cuda:0")
q, k, v, g = (torch.randn(1, 8, 10000, 512, device=dev, dtype=torch.bfloat16) for _ in range(4))
def t(fn, n=30):
    for _ in range(5): fn()
    torch.cuda.synchronize()
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(n): fn()
    b.record(); torch.cuda.synchronize()
    return a.elapsed_time(b) / n
out, lse = ft.fwd(q, k, v, 32, 4, dilated_heads=2)
qa, ka, va = (x[:, :2].contiguous() for x in (q, k, v))
qb, kb, vb = (x[:, 2:].contiguous() for x in (q, k, v))
print("mixed fwd", round(t(lambda: ft.fwd(q, k, v, 32, 4, dilated_heads=2)), 4),
      "A", round(t(lambda: ft.fwd(qa, ka, va, 32, 4)), 4), "B", round(t(lambda: ft.fwd(qb, kb, vb, 32, 1)), 4))
print("mixed bwd", round(t(lambda: ft.bwd(q, k, v, out, lse, g, 32, 4, dilated_heads=2)), 4))
'''
for v in ("1", "0"):
    env = dict(os.environ, FT_WINATTN_MIXED_SERIAL=v)
    r = subprocess.run([sys.executable, "-c", CH], env=env, capture_output=True, text=True)
    print("serial=" + v, r.stdout.strip(), r.stderr[-300:])
