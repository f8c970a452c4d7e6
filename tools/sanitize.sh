#!/bin/bash
# compute-sanitizer passes over small shapes of every kernel family (run under gpurun).
set -u
cd "$(dirname "$0")/.."
cat > /tmp/san_case.py <<'PY'
import os, sys, torch
sys.path.insert(0, ".")
import paper_conf_pldi_tangzwjzyz22_b200 as ft
if len(sys.argv) > 1:   # "nopdl": every launch in plain stream order (FT_KNOB_PDL = 0)
    ft.debug_set("pdl", 0)
from synth import WinAttnShape, make_inputs
dev = torch.device("cuda:0")
for shape, dt in [((1, 2, 300, 64, 32, 3), "bf16"), ((1, 4, 1500, 64, 32, 1), "bf16"),
                  ((1, 2, 700, 64, 20, 5), "bf16"), ((1, 1, 200, 512, 32, 1), "bf16"),
                  ((1, 1, 600, 64, 100, 2), "bf16"), ((1, 1, 500, 128, 80, 1), "bf16"),
                  ((1, 1, 130, 64, 8, 1), "f32"), ((1, 2, 300, 512, 32, 1), "f32"),
                  ((1, 2, 257, 128, 17, 3), "f32"), ((1, 1, 300, 192, 8, 1), "f32"),
                  ((1, 1, 500, 384, 32, 1), "bf16"), ((1, 2, 400, 256, 16, 2), "f32"),   # these two: dS tape
                  ((1, 1, 600, 64, 100, 2), "f32"), ((1, 2, 500, 64, 40, 1), "f32")]:     # fp32 WIDE steps
    s = WinAttnShape(*shape)
    x = make_inputs(s, 0, dt)
    q, k, v, g = (x[n].to(dev) for n in ("q", "k", "v", "dout"))
    o, l = ft.fwd(q, k, v, s.w, s.dilation)
    ft.bwd(q, k, v, o, l, g, s.w, s.dilation)
# dS tape forced below its threshold: bf16 dual-accumulator dK/dV kernel, narrow kernels off
with ft.knobs(dstape=2, narrow=0):
    s = WinAttnShape(1, 2, 500, 128, 32, 1)
    x = make_inputs(s, 0, "bf16")
    q, k, v, g = (x[n].to(dev) for n in ("q", "k", "v", "dout"))
    o, l = ft.fwd(q, k, v, s.w, s.dilation)
    ft.bwd(q, k, v, o, l, g, s.w, s.dilation)
# per-head dilation (ft_winattn_*_mixed)
s = WinAttnShape(1, 4, 400, 64, 16, 3)
x = make_inputs(s, 0, "bf16")
q, k, v, g = (x[n].to(dev) for n in ("q", "k", "v", "dout"))
o, l = ft.fwd(q, k, v, s.w, s.dilation, dilated_heads=2)
ft.bwd(q, k, v, o, l, g, s.w, s.dilation, dilated_heads=2)
# tape path (materialized scores): CUDA-core (fp32) and band tensor-core (bf16) kernels
for dt in ("f32", "bf16"):
    s = WinAttnShape(1, 2, 300, 64, 20, 3)
    x = make_inputs(s, 0, dt)
    q, k, v, g = (x[n].to(dev) for n in ("q", "k", "v", "dout"))
    o, l, tp = ft.fwd_tape(q, k, v, s.w, s.dilation)
    ft.bwd_tape(q, k, v, o, l, tp, g, s.w, s.dilation)
# one-call forward + backward (lse hand-off)
for shape in ((1, 2, 700, 512, 32, 1), (1, 4, 900, 64, 32, 1)):
    s = WinAttnShape(*shape)
    x = make_inputs(s, 0, "bf16")
    q, k, v, g = (x[n].to(dev) for n in ("q", "k", "v", "dout"))
    ft.fwd_bwd(q, k, v, g, s.w, s.dilation)
# SubdivNet circular difference: vector / scalar, gather / scatter, fp32 / bf16
import numpy as np
from paper_conf_pldi_tangzwjzyz22_b200 import subdiv
from synth import mesh_features, torus_mesh
adj = torch.from_numpy(torus_mesh(20, 15, 2).astype(np.int32)).to(dev)
for f, dt in ((64, "f32"), (13, "f32"), (64, "bf16")):
    m = mesh_features(adj.shape[0], f, 0, dt)
    e, dy = m["e"].to(dev), m["dy"].to(dev)
    subdiv.circdiff_fwd(e, adj)
    subdiv.circdiff_bwd(e, adj, dy)
    subdiv.circdiff_bwd(e, adj, dy, symmetric=True)
torch.cuda.synchronize()
print("cases ok")
PY
# one tool per call is the safe pattern on this pool: TOOLS="memcheck" tools/sanitize.sh
for variant in ${VARIANTS:-default nopdl}; do
  for tool in ${TOOLS:-memcheck racecheck synccheck initcheck}; do
    echo "== $tool ($variant)"
    timeout 600 compute-sanitizer --tool $tool --kernel-name kns=tc_ --kernel-name kns=simt --kernel-name kns=circdiff --kernel-name kns=f32_to_bf16 --kernel-name kns=zero_f32 --print-limit 10 \
      python /tmp/san_case.py $([ $variant = nopdl ] && echo nopdl) 2>&1 | tail -4
  done
done
