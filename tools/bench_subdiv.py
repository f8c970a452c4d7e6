"""SubdivNet circular difference on one B200: fwd and bwd throughput and
HBM roofline fraction on synthetic closed torus meshes (synth.torus_mesh), ordered and shuffled.

    python tools/bench_subdiv.py [--nx 1024 --ny 1024 --feats 64 --steps 50]

Algorithmic bytes per face (e = element size, F = n_feats):
  fwd: read e row (F e; the ~3 gathers of a row hit L2 after the first), adj (12); write y (F e)
  bwd: read e row, dy row (2 F e), adj (12); write de (F e)   [+ 4F zeroing / convert passes for
       the fp32 accumulator, counted as overhead]
Inputs (>= 256 MiB of e at the default size) exceed the 126 MiB L2, so no flush is needed.
Prints one JSON line per (dtype, ordering).
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
import paper_conf_pldi_tangzwjzyz22_b200 as ft  # noqa: E402
from paper_conf_pldi_tangzwjzyz22_b200 import subdiv  # noqa: E402
from synth import torus_mesh  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--nx", type=int, default=1024)
    ap.add_argument("--ny", type=int, default=1024)
    ap.add_argument("--feats", type=int, default=64)
    ap.add_argument("--steps", type=int, default=50)
    a = ap.parse_args()
    dev = torch.device("cuda:0")
    hbm_peak = bench.load_peaks()[0]
    for shuffle in (None, 7):
        adj_np = torus_mesh(a.nx, a.ny, shuffle)
        n = adj_np.shape[0]
        adj = torch.from_numpy(adj_np.astype(np.int32)).to(dev)
        for dt in (torch.float32, torch.bfloat16):
            e = (torch.rand(n, a.feats, device=dev) * 2 - 1).to(dt)
            dy = (torch.rand(n, a.feats, device=dev) * 2 - 1).to(dt)
            y, de = torch.empty_like(e), torch.empty_like(e)
            es = e.element_size()
            for _ in range(3):
                subdiv.circdiff_fwd(e, adj, y)
                subdiv.circdiff_bwd(e, adj, dy, de)
                subdiv.circdiff_bwd(e, adj, dy, de, symmetric=True)
            torch.cuda.synchronize()
            res = {"workload": "subdivnet_circdiff", "faces": n, "feats": a.feats,
                   "dtype": "f32" if dt == torch.float32 else "bf16",
                   "mesh": f"torus {a.nx}x{a.ny}" + (" shuffled" if shuffle is not None else " ordered")}
            for name, fn, alg in (("fwd", lambda: subdiv.circdiff_fwd(e, adj, y), n * (2 * a.feats * es + 12)),
                                  ("bwd_scatter", lambda: subdiv.circdiff_bwd(e, adj, dy, de), n * (3 * a.feats * es + 12)),
                                  ("bwd_gather", lambda: subdiv.circdiff_bwd(e, adj, dy, de, symmetric=True),
                                   n * (3 * a.feats * es + 12))):
                evs = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
                evs[0].record()
                for _ in range(a.steps):
                    fn()
                evs[1].record()
                torch.cuda.synchronize()
                ms = evs[0].elapsed_time(evs[1]) / a.steps
                gbs = alg / (ms / 1e3) / 1e9
                res[name] = {"ms": ms, "faces_per_s": n / (ms / 1e3), "algorithmic_bytes": alg,
                             "achieved_gbs": gbs, "hbm_frac": gbs / hbm_peak}
            res["hbm_peak_gbs"] = hbm_peak
            print(json.dumps(res), flush=True)


if __name__ == "__main__":
    main()
