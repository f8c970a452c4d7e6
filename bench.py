#!/usr/bin/env python
"""bench.py -- fwd+bwd banded window-attention throughput on B200 (one JSON line).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--workload C2a] [--dtype f32|bf16]
    python -m torch.distributed.run --nproc-per-node N --master-addr 127.0.0.1 ... bench.py --gpus N
    python bench.py --impl reference ...      # the fp64 CPU oracle as the reference arm

A step is one pass of the whole hot path (SURVEY.md §8(a) F0-F6 + B0-B5): ft_winattn_fwd
then ft_winattn_bwd over one batch of synthetic inputs resident in HBM.  Default workload
is BASELINE.json configs[2] "same shape forward+backward" at reading A14(a) of the
paper's Longformer shape: B=1, H=8, L=10000, d=512, w=32 (C2a), in fp32 -- the paper's
precision ("f32"), computed on the tensor cores as bf16 hi / lo planes
within the north_star's 1e-4 bound (csrc/tc_band32.cu).  --dtype bf16 measures bf16 storage.

Multi-GPU: (batch, head) units are independent, so the job is sharded
with NO collective on the data path: every rank runs its own batch element (weak scaling,
global_batch = N), timed between a barrier + synchronize on both sides, and the elapsed
time is the max over ranks.  The "strong_scaling" record splits the fixed --strong-workload
(64 heads of 32K tokens by default) into per-rank head slabs; "e2e_nccl_scatter_gather" adds
the NCCL scatter of the inputs and gather of the outputs from rank 0.

Keys beyond the base contract: "roofline" (dominant kernel, CUDA events on the launching
stream via the ft_winattn_profile_events hook, recorded in a second pass of the same steps:
an event between two launches would stop the BWDQ -> BWDKV programmatic dependent launch
overlap inside the timed region), "hbm_step" (whole step vs SURVEY.md §8(d)
algorithmic bytes), "cpu_baseline" (the fp64 oracle on a bounded sample, rank 0, N=1),
"e2e" (pinned host buffers, H2D + fwd + bwd + D2H inside the timed region), "clocks"
(NVML samples during the timed region), "gpu_launches", and the sub-records "bf16" / "f32"
(the other storage dtype), "fwd_bwd_call" (the one-call API), "strong_scaling" and, at N = 1,
"other_configs" (every other BASELINE configuration timed in the same run).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

WORKLOADS = {
    # name: (batch per rank, heads, seq_len, d, w, dilation, description)
    "C2a": (1, 8, 10000, 512, 32, 1, "BASELINE configs[2]: Longformer-shaped fwd+bwd, reading A14(a)"),
    "C2a_dil": (1, 2, 10000, 512, 32, 4, "C2a's dilated heads (artefact heads 0-1, dilation 4)"),
    "C2b": (1, 12, 4096, 64, 256, 1, "Longformer-base shape, reading A14(b)"),
    "C4d2": (1, 12, 16384, 64, 256, 2, "BASELINE configs[3]: dilated w=256, 16K tokens"),
    "C4d4": (1, 12, 16384, 64, 256, 4, "BASELINE configs[3]: dilated w=256, 16K tokens"),
    "C5_w32": (1, 64, 32768, 64, 32, 1, "BASELINE configs[4] sweep corner, HBM-bound"),
    "C5_w256": (1, 64, 32768, 64, 256, 1, "BASELINE configs[4] sweep corner, ridge"),
    "C5_small": (1, 8, 4096, 64, 32, 1, "BASELINE configs[4] sweep corner, small"),
    # per-head dilation in one call (ft_winattn_*_mixed): heads 0-1 dilation 4, heads 2-7 dilation 1
    "C2a_mix": (1, 8, 10000, 512, 32, 4, "C2a with the artefact's mixed heads (0-1 dilated x4), one call", 2),
}

METRIC = "window-attn fwd+bwd tokens/s per GPU and % HBM roofline at 1/2/4/8 B200"
L2_BYTES = 126 * 1024 * 1024


def load_peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            p = json.load(f)
        return float(p["hbm_gbs"]), float(p["bf16_tflops"]), float(p.get("sm_max_mhz", 1965.0)), "measured"
    except Exception:
        return 6650.0, 1590.0, 1965.0, "fallback"


# ----------------------------------------------------------------------------- algorithmic work
def rows_of(B, H, L):
    return B * H * L


def window_sizes(L, w, dil):
    """n_i = |N(i)| for every row (SURVEY.md §8 closed form, pinned by the oracle tests)."""
    import numpy as np
    i = np.arange(L)
    return np.minimum(w, i // dil) + np.minimum(w, (L - 1 - i) // dil) + 1


def kernel_bytes_per_row(kind: str, d: int, e: int) -> int:
    """Minimal HBM bytes one row of each kernel must move.
    fwd : read q, k, v ; write o (dtype) and lse (fp32)                 = 4de + 4
    bwdA: read q, k, v, dout, lse ; write dq, D                          = 5de + 8
    bwdB: read q, k, v, dout, lse, D ; write dk, dv                      = 6de + 8
    rowdot (wide windows): read dout, o ; write D                        = 2de + 4"""
    return {"fwd": 4 * d * e + 4, "bwdA": 5 * d * e + 8, "bwdB": 6 * d * e + 8,
            "rowdot": 2 * d * e + 4}[kind]


def step_bytes_per_row(d: int, e: int) -> int:
    """fwd 4de+4 plus bwd 8de+4 (the bwd figure counts reading o)."""
    return (4 * d * e + 4) + (8 * d * e + 4)


def launch_table(ft, B, H, L, d, w, dil, code):
    """[(kind, rows)] of the forward and backward launches of one call, in launch order, with the
    rows each launch processes (launches cover residue groups of 8 -- 4 for the wide-window
    kernels -- of the min(dil, L) residues)."""
    path_f, nf = ft.plan(False, B, H, L, d, w, dil, code)
    path_b, nb = ft.plan(True, B, H, L, d, w, dil, code)
    rows = rows_of(B, H, L)
    nres = min(dil, L)

    def split(n_launch, res_per):
        sizes = [min(res_per, nres - i) for i in range(0, nres, res_per)]
        if len(sizes) != n_launch:   # SIMT kernels and anything else: every launch sees all rows
            return [rows] * n_launch
        return [rows * sz / nres for sz in sizes]

    res = 8 if (min(w, L) <= 64 or code == 0) else 4   # fp32 tensor-core launches: 8 residues
    fwd = [("fwd", r) for r in (split(nf, res) if path_f == ft.PATH_TC else [rows] * nf)]
    if path_b == ft.PATH_TC:
        pre = nb % 2                                     # wide windows: optional rowdot pre-pass
        g = (nb - pre) // 2
        per = split(g, res)
        bwd = [("rowdot", rows)] * pre + [("bwdA", r) for r in per] + [("bwdB", r) for r in per]
    else:
        bwd = [("bwdA", rows)] + [("bwdB", rows)] * (nb - 1)
    return path_f, path_b, fwd, bwd


# ----------------------------------------------------------------------------- clocks (NVML)
class ClockSampler:
    REASONS = {
        0x1: "gpu_idle", 0x2: "applications_clocks_setting", 0x4: "sw_power_cap",
        0x8: "hw_slowdown", 0x10: "sync_boost", 0x20: "sw_thermal_slowdown",
        0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown", 0x100: "display_clock_setting",
    }

    def __init__(self, index: int, period_s: float = 0.001):
        self.index, self.period = index, period_s
        self.samples, self.reasons = [], set()
        self._stop = threading.Event()
        self.ok = False
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
            self.ok = True
        except Exception:
            self.max_mhz = None

    def _run(self):
        nv = self.nv
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksThrottleReasons(self.h)
                for bit, name in self.REASONS.items():
                    if r & bit and bit != 0x1:
                        self.reasons.add(name)
            except Exception:
                pass
            time.sleep(self.period)

    def __enter__(self):
        if self.ok:
            self.t = threading.Thread(target=self._run, daemon=True)
            self.t.start()
        return self

    def __exit__(self, *a):
        if self.ok:
            self._stop.set()
            self.t.join()

    def summary(self):
        if not self.ok or not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons),
                    "samples": len(self.samples)}
        return {"sm_mhz": statistics.median(self.samples), "sm_max_mhz": self.max_mhz,
                "reasons": sorted(self.reasons), "samples": len(self.samples)}


# ----------------------------------------------------------------------------- CPU oracle legs
def oracle_sample(shape, units: int, rows_cap: int, seed: int = 0):
    """Time the fp64 oracle fwd+bwd on `units` (batch, head) units of the workload, each
    truncated to its first rows_cap rows (its own band problem; per-row work equals the
    full problem's away from the two sequence edges).  Returns (seconds, units, rows)."""
    import numpy as np
    import oracle
    B, H, L, d, w, dil = shape
    Ls = min(L, rows_cap)
    rng = np.random.Generator(np.random.PCG64(seed))
    x = [rng.uniform(-1.0, 1.0, size=(1, units, Ls, d)) for _ in range(4)]
    oracle.fwd(x[0][:, :1, :8], x[1][:, :1, :8], x[2][:, :1, :8], w, dil)   # load / warm
    t0 = time.perf_counter()
    o, lse = oracle.fwd(x[0], x[1], x[2], w, dil)
    oracle.bwd(x[0], x[1], x[2], o, lse, x[3], w, dil)
    return time.perf_counter() - t0, units, Ls


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_baseline(shape, budget_s: float = 15.0):
    """The oracle as it stands, on as many whole (batch, head) units of the workload as fit
    in ~budget_s seconds of CPU work (at least one unit), extrapolated per unit."""
    import oracle
    B, H, L, d, w, dil = shape
    s1, _, Ls = oracle_sample(shape, 1, L)
    n = int(max(1, min(B * H, budget_s // max(s1, 1e-3))))
    secs, n, Ls = oracle_sample(shape, n, L, seed=1) if n > 1 else (s1, 1, Ls)
    # the whole workload takes less than the budget: repeat whole passes (~budget_s in total)
    reps = 1
    if n == B * H and secs < budget_s / 2:
        extra = int(budget_s // max(secs, 1e-3)) - 1
        for r in range(extra):
            secs += oracle_sample(shape, n, L, seed=2 + r)[0]
        reps += extra
    value = reps * (n * Ls / secs) / (B * H) * B
    return {"value": value, "unit": "tokens/s", "cores": oracle.num_threads(), "kind": "oracle",
            "cpu_model": cpu_model(),
            "sample": f"fp64 oracle fwd+bwd on {n} of {B * H} (batch, head) units at full length "
                      f"{Ls}, {reps} pass(es); {secs:.2f} s of CPU work; tokens/s extrapolated "
                      f"linearly per unit",
            "seconds": secs}


def run_reference(args, shape, cfg):
    """--impl reference: the fp64 CPU oracle as it stands, rank 0 only."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    B, H, L, d, w, dil = shape
    rows_cap = args.ref_rows if args.ref_rows > 0 else L
    for _ in range(args.warmup):
        oracle_sample(shape, 1, rows_cap)
    times = []
    Ls = rows_cap
    for _ in range(args.steps):
        s, _, Ls = oracle_sample(shape, 1, rows_cap)
        times.append(s)
    mean = sum(times) / len(times)
    value = (Ls / mean) / (B * H) * B
    line = {
        "impl": "reference", "metric": METRIC, "value": value, "unit": "tokens/s",
        "n_gpus": args.gpus, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": mean * 1e3, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic", "config": cfg,
        "cpu_baseline": {"value": value, "unit": "tokens/s", "kind": "oracle",
                         "cores": oracle.num_threads(),
                                  "sample": f"each step: fp64 oracle fwd+bwd on 1 of {B * H} (batch, head) "
                                   f"units, {Ls} of {L} rows, tokens/s extrapolated per unit"},
        "e2e": {"value": value, "unit": "tokens/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }
    print(json.dumps(line), flush=True)


# ----------------------------------------------------------------------------- GPU arm
def scatter_gather_e2e(args, rank, world, dev, tdt, e, shape):
    """N > 1: the north_star's end-to-end multi-GPU variant (dist.sharded_fwd_bwd).  Rank 0 owns
    the full [B*N, H, L, d] tensors, scatters (batch, head) slabs with NCCL, every rank runs
    fwd+bwd on its slab, and out / lse / dq / dk / dv are gathered back.  CUDA events between
    barriers, max over ranks."""
    import torch
    import torch.distributed as dist
    from paper_conf_pldi_tangzwjzyz22_b200.dist import sharded_fwd_bwd
    B, H, L, d, w, dil = shape
    full = [None] * 4
    if rank == 0:
        gen0 = torch.Generator(device=dev)
        gen0.manual_seed(99)
        full = [(torch.rand((B * world, H, L, d), device=dev, generator=gen0) * 2 - 1).to(tdt)
                for _ in range(4)]
    run = lambda: sharded_fwd_bwd(*full, w, dil, shape=(B * world, H, L, d), dtype=tdt, device=dev)  # noqa: E731
    run()   # warm-up
    torch.cuda.synchronize()
    dist.barrier()
    a0, a1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a0.record()
    for _ in range(args.sg_steps):
        run()
    a1.record()
    torch.cuda.synchronize()
    t = torch.tensor([a0.elapsed_time(a1) / args.sg_steps], device=dev, dtype=torch.float64)
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t.item())
    n_el = B * world * H * L * d
    return {"value": B * world * L / (ms / 1e3), "unit": "tokens/s", "ms_per_step": ms,
            "steps": args.sg_steps, "bytes_scattered": 4 * n_el * e,
            "bytes_gathered": 4 * n_el * e + B * world * H * L * 4,
            "what": "rank 0 scatters q/k/v/dout (NCCL), per-rank fwd+bwd, gathers out/lse/dq/dk/dv"}


def quick_time(ft, torch, dev, shape, dtype, steps, warmup, hd=None, api="separate", units=None):
    """ms per fwd+bwd step of `shape` (B, H, L, d, w, dil) on this rank: inputs generated on the
    device, L2 flushed between steps when they fit in it, CUDA events around the K steps.
    api: "separate" = ft_winattn_fwd + ft_winattn_bwd, "fwd_bwd" = the one-call ft_winattn_fwd_bwd.
    units: heads of this rank's slab (strong scaling), default H."""
    B, H, L, d, w, dil = shape
    H = H if units is None else units
    tdt = torch.bfloat16 if dtype == "bf16" else torch.float32
    e = 2 if dtype == "bf16" else 4
    gen = torch.Generator(device=dev)
    gen.manual_seed(4321)
    q, k, v, g = ((torch.rand((B, H, L, d), device=dev, generator=gen) * 2 - 1).to(tdt) for _ in range(4))
    out, dq, dk, dv = (torch.empty_like(q) for _ in range(4))
    lse = torch.empty((B, H, L), device=dev, dtype=torch.float32)
    ws = torch.empty(max(ft.workspace_bytes(q, w, dil), 16), device=dev, dtype=torch.uint8)
    flush = torch.empty(2 * L2_BYTES, device=dev, dtype=torch.uint8) if 4 * q.numel() * e <= L2_BYTES else None

    def step():
        if api == "fwd_bwd":
            ft.fwd_bwd(q, k, v, g, w, dil, out=out, lse=lse, dq=dq, dk=dk, dv=dv, workspace=ws)
        else:
            ft.fwd(q, k, v, w, dil, out=out, lse=lse, dilated_heads=hd)
            ft.bwd(q, k, v, out, lse, g, w, dil, dq=dq, dk=dk, dv=dv, workspace=ws, dilated_heads=hd)

    for _ in range(warmup):
        step()
    torch.cuda.synchronize()
    tot = 0.0
    for _ in range(steps):
        if flush is not None:
            flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        step()
        b.record()
        b.synchronize()
        tot += a.elapsed_time(b)
    return tot / steps


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=10)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="C2a", choices=sorted(WORKLOADS))
    ap.add_argument("--dtype", default="f32", choices=["bf16", "f32"],
                    help="f32: the paper's precision (PAPER.md:147, 217), the headline; bf16: faster storage")
    ap.add_argument("--strong-workload", default="C5_w32",
                    help="fixed-work (batch, head)-sharded strong-scaling record (configs[4] corner)")
    ap.add_argument("--extra-steps", type=int, default=50, help="steps of each sub-record")
    ap.add_argument("--no-extras", action="store_true", help="skip the sub-records")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=15.0, help="seconds of oracle work (cpu_baseline)")
    ap.add_argument("--ref-rows", type=int, default=0, help="oracle rows per reference step (0 = full L)")
    ap.add_argument("--e2e-steps", type=int, default=20)
    ap.add_argument("--sg-steps", type=int, default=3, help="N > 1: NCCL scatter/gather end-to-end steps")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    B, H, L, d, w, dil, desc = WORKLOADS[args.workload][:7]
    hd = WORKLOADS[args.workload][7] if len(WORKLOADS[args.workload]) > 7 else None
    world = int(os.environ.get("WORLD_SIZE", "1"))
    shape = (B, H, L, d, w, dil)
    e = 2 if args.dtype == "bf16" else 4
    in_bytes = 4 * B * H * L * d * e
    cfg = {"workload": args.workload, "desc": desc, "batch_per_rank": B, "heads": H, "seq_len": L,
           "d": d, "w": w, "dilation": dil, "global_batch": B * world,
           **({"dilated_heads": hd} if hd is not None else {}),
           "parallelism": f"dp{world} over (batch, head) units, no collective on the data path",
           "l2": ("inputs larger than L2" if in_bytes > L2_BYTES else "L2 flushed between steps") +
                 f" ({in_bytes / 2**20:.0f} MiB of q/k/v/dout vs {L2_BYTES / 2**20:.0f} MiB L2)"}
    if args.impl == "reference":
        run_reference(args, shape, cfg)
        return

    import torch
    import torch.distributed as dist
    import paper_conf_pldi_tangzwjzyz22_b200 as ft

    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    # FT_BENCH_ONE_GPU=1 (self-test of the multi-rank code path on a one-GPU box): every rank
    # uses cuda:0 and the gloo backend (NCCL refuses two ranks on one device).  Not for timing.
    one_gpu = os.environ.get("FT_BENCH_ONE_GPU") == "1"
    if one_gpu:
        local_rank = 0
    if world > 1:
        torch.cuda.set_device(local_rank)
        if one_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    ft.load_library()
    tdt = torch.bfloat16 if args.dtype == "bf16" else torch.float32
    code = ft.FT_BF16 if args.dtype == "bf16" else ft.FT_F32
    if hd is None:
        path_f, path_b, ltf, ltb = launch_table(ft, B, H, L, d, w, dil, code)
    else:   # B = 1: the dilated head slice, then the rest (ft_winattn_*_mixed launch order)
        assert B == 1
        ltf, ltb = [], []
        for nh, dl in ((hd, dil), (H - hd, 1)):
            if nh:
                path_f, path_b, f_, b_ = launch_table(ft, 1, nh, L, d, w, dl, code)
                ltf += f_
                ltb += b_
    nf, nb = len(ltf), len(ltb)

    gen = torch.Generator(device=dev)
    gen.manual_seed(1234 + rank)
    def rnd():
        return (torch.rand((B, H, L, d), device=dev, generator=gen, dtype=torch.float32) * 2 - 1).to(tdt)
    q, k, v, g = rnd(), rnd(), rnd(), rnd()
    out, dq, dk, dv = (torch.empty_like(q) for _ in range(4))
    lse = torch.empty((B, H, L), device=dev, dtype=torch.float32)
    ws = torch.empty(max(ft.workspace_bytes(q, w, dil), 16), device=dev, dtype=torch.uint8)
    flush = None
    if in_bytes <= L2_BYTES:
        flush = torch.empty(2 * L2_BYTES, device=dev, dtype=torch.uint8)

    def step():
        ft.fwd(q, k, v, w, dil, out=out, lse=lse, dilated_heads=hd)
        ft.bwd(q, k, v, out, lse, g, w, dil, dq=dq, dk=dk, dv=dv, workspace=ws, dilated_heads=hd)

    for _ in range(args.warmup):
        step()
    torch.cuda.synchronize()

    # ---------------------------------------------------------------- timed region
    stream = torch.cuda.current_stream(dev)
    def ev():
        e_ = torch.cuda.Event(enable_timing=True)
        e_.record(stream)   # materialise the CUDA event so its handle can go through the ABI
        return e_
    starts, ends = [], []
    sampler = ClockSampler(dev.index if dev.index is not None else 0)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with sampler:
        for _ in range(args.steps):
            if flush is not None:
                flush.zero_()   # outside the events: evicts q/k/v/dout from L2
            s0, s1 = ev(), ev()
            s0.record(stream)
            step()
            s1.record(stream)
            starts.append(s0); ends.append(s1)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    step_ms = [a.elapsed_time(b) for a, b in zip(starts, ends)]
    elapsed_ms = sum(step_ms)
    # Per-kernel durations: a second pass over the same steps with an event recorded after
    # every launch (each launch timed from the previous event on the same stream).  It is
    # kept out of the timed region because an event between two launches stops the
    # programmatic-dependent-launch overlap (BWDQ -> BWDKV): these durations are serialised,
    # i.e. conservative for the roofline.
    names = [f"fwd{i}" for i in range(nf)] + [f"bwd{i}" for i in range(nb)]
    kdur = {n: [] for n in names}
    kpass = min(args.steps, 50)
    rec = []
    # a mixed call runs its head groups on two streams; events chained across them would not
    # time one launch each, so this pass enqueues every launch on the timed stream
    serial = ft.knobs(side=0)
    serial.__enter__()
    for _ in range(kpass):
        if flush is not None:
            flush.zero_()
        s0, fe, be = ev(), [ev() for _ in range(nf)], [ev() for _ in range(nb)]
        s0.record(stream)
        with ft.profile_events(fe):
            ft.fwd(q, k, v, w, dil, out=out, lse=lse, dilated_heads=hd)
        with ft.profile_events(be):
            ft.bwd(q, k, v, out, lse, g, w, dil, dq=dq, dk=dk, dv=dv, workspace=ws, dilated_heads=hd)
        rec.append((s0, fe, be))
    torch.cuda.synchronize()
    serial.__exit__()
    for s0, fe, be in rec:
        prev = s0
        for n, e1 in zip(names, fe + be):
            kdur[n].append(prev.elapsed_time(e1))
            prev = e1
    if world > 1:
        t = torch.tensor([elapsed_ms], device="cpu" if one_gpu else dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        elapsed_ms = float(t.item())

    tokens = B * L * world * args.steps
    value = tokens / (elapsed_ms / 1e3)
    hbm_peak, bf16_peak, sm_max, peak_src = load_peaks()
    rows = rows_of(B, H, L)

    # dominant kernel roofline (kind and rows of every launch: launch_table)
    kinds = {f"fwd{i}": kd for i, (kd, _) in enumerate(ltf)}
    kinds.update({f"bwd{i}": kd for i, (kd, _) in enumerate(ltb)})
    krows = {f"fwd{i}": r for i, (_, r) in enumerate(ltf)}
    krows.update({f"bwd{i}": r for i, (_, r) in enumerate(ltb)})
    mean_k = {n: sum(x) / len(x) for n, x in kdur.items()}
    dom = max(mean_k, key=mean_k.get)
    # The roofline is taken over the direction (forward or backward) whose launches take the most
    # time, with SURVEY.md §8(d)'s algorithmic bytes of that direction -- fwd 4de + 4, bwd 8de + 4
    # per row -- over the sum of its launches' CUDA-event durations.  (Round 1 booked the dominant
    # launch's own I/O, e.g. the dK/dV kernel's 6de + 8, which flattered it.)  per_kernel adds each
    # launch's own-I/O figure for detail.
    t_dir = {"fwd": sum(v for n, v in mean_k.items() if n.startswith("fwd")),
             "bwd": sum(v for n, v in mean_k.items() if n.startswith("bwd"))}
    ddir = max(t_dir, key=t_dir.get)
    per_kernel = {n: {"kind": kinds[n], "ms": mean_k[n],
                      "own_io_gbs": kernel_bytes_per_row(kinds[n], d, e) * krows[n] / (mean_k[n] / 1e3) / 1e9}
                  for n in mean_k}
    if path_b == ft.PATH_TC:   # tensor-core kernels (bf16, or fp32 as bf16 hi / lo planes): HBM bound
        by = ((4 if ddir == "fwd" else 8) * d * e + 4) * rows
        ach = by / (t_dir[ddir] / 1e3) / 1e9
        roof = {"bound": "hbm", "achieved": ach, "peak": hbm_peak, "unit": "GB/s",
                "frac": ach / hbm_peak, "traffic": None, "kernel": f"{ddir} ({', '.join(n for n in mean_k if n.startswith(ddir))})",
                "ms_per_launch": t_dir[ddir], "algorithmic_bytes_per_launch": by,
                "algorithmic_bytes_rule": "SURVEY.md §8(d): fwd 4de+4, bwd 8de+4 per row",
                "peak_source": peak_src, "per_kernel": per_kernel}
    else:
        nsum = float(window_sizes(L, w, dil).sum()) * B * H
        fl = {"fwd": 4, "bwdA": 6, "bwdB": 8}[kinds[dom]] * d * nsum
        ach = fl / (mean_k[dom] / 1e3) / 1e12
        fma_peak = 148 * 128 * 2 * sm_max * 1e6 / 1e12
        roof = {"bound": "alu", "achieved": ach, "peak": fma_peak, "unit": "TFLOP/s",
                "frac": ach / fma_peak, "traffic": None, "kernel": dom, "kernel_kind": kinds[dom],
                "ms_per_launch": mean_k[dom],
                "peak_source": "derived: 148 SM x 128 FP32 lanes x 2 flop x sm_max_mhz"}
    tr_path = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tr_path):
        try:
            trj = json.load(open(tr_path))
            if path_b == ft.PATH_TC:   # DRAM bytes of the direction's launches (ncu --set full)
                names = [n for n in mean_k if n.startswith(ddir)]
                trs = [trj.get(f"{args.workload}/{args.dtype}/{kinds[n]}") for n in names]
                if trs and all(trs):
                    roof["traffic"] = sum(t["bytes_per_launch"] for t in trs)
                    roof["traffic_source"] = trs[0].get("source")
            else:
                tr = trj.get(f"{args.workload}/{args.dtype}/{kinds[dom]}")
                if tr:
                    roof["traffic"] = tr["bytes_per_launch"]
                    roof["traffic_source"] = tr.get("source")
        except Exception:
            pass
    step_alg = step_bytes_per_row(d, e) * rows * world
    hbm_step = {"algorithmic_bytes_per_step": step_alg,
                "achieved_gbs": step_alg / (elapsed_ms / args.steps / 1e3) / 1e9 / world,
                "peak": hbm_peak, "frac": step_alg / (elapsed_ms / args.steps / 1e3) / 1e9 / world / hbm_peak}
    # the step against every ceiling of SURVEY.md §8(d): HBM bytes, tensor (bf16) or FMA (fp32)
    # flops (fwd 4 d n_i + bwd 8 d n_i per row), MUFU ex2 (n_i per row in each direction); the
    # binding ceiling is the one with the largest lower-bound time
    step_s = elapsed_ms / args.steps / 1e3
    nsum = float(window_sizes(L, w, dil).sum()) * B * H
    flops = 12.0 * d * nsum
    exps = 2.0 * nsum
    sm_mhz = sm_max
    # the tensor ceiling: bf16 products at the measured bf16 peak; the fp32 tensor-core path issues
    # three bf16 products (hi.hi + hi.lo + lo.hi) per fp32 product; the CUDA-core path: FMA
    tc_path = path_b == ft.PATH_TC
    comp_peak = bf16_peak * 1e12 if tc_path else 148 * 128 * 2 * sm_mhz * 1e6
    comp_work = flops * (3.0 if (tc_path and args.dtype == "f32") else 1.0)
    mufu_peak = 148 * 16 * sm_mhz * 1e6
    bounds = {"hbm": step_alg / world / (hbm_peak * 1e9), "tensor" if tc_path else "fma": comp_work / comp_peak,
              "mufu": exps / mufu_peak}
    ceilings = {k: {"lower_bound_us": v * 1e6, "frac": v / step_s} for k, v in bounds.items()}
    ceilings["binding"] = max(bounds, key=bounds.get)
    ceilings["peaks"] = {"hbm_gbs": hbm_peak, "compute_tflops": comp_peak / 1e12, "mufu_gops": mufu_peak / 1e9,
                         "note": "HBM and bf16 measured (MEASURED_PEAKS.json); FMA and MUFU derived from "
                                 "148 SMs x 128 lanes x 2 / 16 ex2 per clock at sm_max_mhz; fp32 on the "
                                 "tensor cores counts 3 bf16 products per fp32 product"}
    ceilings["step_ms"] = {"mean": elapsed_ms / args.steps, "min": min(step_ms),
                           "median": sorted(step_ms)[len(step_ms) // 2]}

    # ---------------------------------------------------------------- e2e (pinned host buffers)
    # Every step copies its inputs host -> device, runs fwd + bwd through the public API and
    # copies its results device -> host, all inside the timed region.  The steps are
    # pipelined the way a serving loop would be: two device buffer sets, H2D on one stream,
    # compute on another, D2H on a third, so step i+1's inputs and step i-1's results cross
    # PCIe (full duplex) while step i computes.
    e2e = None
    if args.e2e_steps > 0:
        hq, hk, hv, hg = (x.cpu().pin_memory() for x in (q, k, v, g))
        ho, hdq, hdk, hdv = (torch.empty_like(hq).pin_memory() for _ in range(4))
        hl = torch.empty(lse.shape, dtype=torch.float32).pin_memory()
        sets = [(q, k, v, g, out, lse, dq, dk, dv, ws)]
        sets.append(tuple(torch.empty_like(t) for t in sets[0]))
        s_in, s_cmp, s_out = (torch.cuda.Stream(dev) for _ in range(3))
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        mk = lambda: torch.cuda.Event(enable_timing=True)  # noqa: E731
        e0, e1 = mk(), mk()
        n = args.e2e_steps
        h2d_done = [torch.cuda.Event() for _ in range(n)]
        cmp_done = [torch.cuda.Event() for _ in range(n)]
        d2h_done = [torch.cuda.Event() for _ in range(n)]
        e0.record(s_in)
        s_cmp.wait_event(e0)
        s_out.wait_event(e0)
        for i in range(n):
            tq, tk, tv, tg, to, tl, tdq, tdk, tdv, tws = sets[i % 2]
            with torch.cuda.stream(s_in):
                if i >= 2:
                    s_in.wait_event(cmp_done[i - 2])   # set i%2's inputs were read by step i-2
                for dst, src in ((tq, hq), (tk, hk), (tv, hv), (tg, hg)):
                    dst.copy_(src, non_blocking=True)
                h2d_done[i].record(s_in)
            with torch.cuda.stream(s_cmp):
                s_cmp.wait_event(h2d_done[i])
                if i >= 2:
                    s_cmp.wait_event(d2h_done[i - 2])   # set i%2's results were read back
                ft.fwd(tq, tk, tv, w, dil, out=to, lse=tl, dilated_heads=hd)
                ft.bwd(tq, tk, tv, to, tl, tg, w, dil, dq=tdq, dk=tdk, dv=tdv, workspace=tws,
                       dilated_heads=hd)
                cmp_done[i].record(s_cmp)
            with torch.cuda.stream(s_out):
                s_out.wait_event(cmp_done[i])
                for dst, src in ((ho, to), (hl, tl), (hdq, tdq), (hdk, tdk), (hdv, tdv)):
                    dst.copy_(src, non_blocking=True)
                d2h_done[i].record(s_out)
        s_out.wait_event(h2d_done[n - 1])
        e1.record(s_out)
        torch.cuda.synchronize()
        ems = e0.elapsed_time(e1)
        if world > 1:
            t = torch.tensor([ems], device="cpu" if one_gpu else dev, dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            ems = float(t.item())
        e2e = {"value": B * L * world * args.e2e_steps / (ems / 1e3), "unit": "tokens/s",
               "h2d_bytes_per_step": 4 * q.numel() * e,
               "d2h_bytes_per_step": 4 * q.numel() * e + lse.numel() * 4,
               "steps": args.e2e_steps, "pipelined": "2 buffer sets; H2D / compute / D2H streams"}

    # ---------------------------------------------------------------- N > 1: NCCL scatter / gather
    # The north_star's end-to-end multi-GPU variant (dist.sharded_fwd_bwd): rank 0 owns the full
    # [B*N, H, L, d] tensors, scatters (batch, head) slabs over NVLink, every rank runs fwd+bwd on
    # its slab, and out / lse / dq / dk / dv are gathered back.  Timed with CUDA events between
    # barriers, max over ranks.  Not in one_gpu self-test mode (gloo has no CUDA scatter).
    sg = None
    if world > 1 and not one_gpu and args.sg_steps > 0:
        try:
            sg = scatter_gather_e2e(args, rank, world, dev, tdt, e, (B, H, L, d, w, dil))
        except Exception as ex:   # the main line must survive; report why this extra is missing
            sg = {"error": f"{type(ex).__name__}: {ex}"[:300]}

    # ---------------------------------------------------------------- sub-records
    # (a) the other storage dtype on the same workload; (b) the one-call ft_winattn_fwd_bwd (the
    # forward -> dQ-kernel lse hand-off); (c) fixed-work strong scaling: the --strong-workload's
    # (batch, head) units split into contiguous slabs over the N ranks (rank r
    # owns [r U / N, (r + 1) U / N)), compute only, max over ranks; the NCCL scatter / gather
    # variant of the same job is e2e_nccl_scatter_gather.
    extras = {}
    if not args.no_extras and args.extra_steps > 0:
        other = "bf16" if args.dtype == "f32" else "f32"
        o_ms = quick_time(ft, torch, dev, shape, other, args.extra_steps, 3, hd=hd)
        oe = 2 if other == "bf16" else 4
        o_ms_t = torch.tensor([o_ms], dtype=torch.float64, device="cpu" if one_gpu else dev)
        if world > 1:
            dist.all_reduce(o_ms_t, op=dist.ReduceOp.MAX)
        o_ms = float(o_ms_t.item())
        extras[other] = {"ms_per_step": o_ms, "tokens_per_s": B * L * world / (o_ms / 1e3),
                         "hbm_frac": step_bytes_per_row(d, oe) * rows / (o_ms / 1e3) / 1e9 / hbm_peak,
                         "paths": dict(zip(("fwd", "bwd"), ("tc" if ft.plan(b_, B, H, L, d, w, dil,
                                                                      ft.FT_BF16 if other == "bf16" else ft.FT_F32)[0]
                                                   == ft.PATH_TC else "simt" for b_ in (False, True))))}
        if hd is None:
            fb_ms = quick_time(ft, torch, dev, shape, args.dtype, args.extra_steps, 3, api="fwd_bwd")
            fb_t = torch.tensor([fb_ms], dtype=torch.float64, device="cpu" if one_gpu else dev)
            if world > 1:
                dist.all_reduce(fb_t, op=dist.ReduceOp.MAX)
            fb_ms = float(fb_t.item())
            extras["fwd_bwd_call"] = {"ms_per_step": fb_ms, "tokens_per_s": B * L * world / (fb_ms / 1e3),
                                      "what": "ft_winattn_fwd_bwd: one call, the dQ kernel reads lse rows as "
                                              "the forward stores them"}
        sw = WORKLOADS[args.strong_workload]
        sB, sH, sL, sd, sw_, sdil = sw[:6]
        U = sB * sH
        u0, u1 = (rank * U) // world, ((rank + 1) * U) // world
        if sB == 1 and u1 > u0:
            s_ms = quick_time(ft, torch, dev, (1, sH, sL, sd, sw_, sdil), args.dtype, args.extra_steps, 3,
                              units=u1 - u0)
        else:
            s_ms = 0.0
        s_t = torch.tensor([s_ms], dtype=torch.float64, device="cpu" if one_gpu else dev)
        if world > 1:
            dist.barrier()
            dist.all_reduce(s_t, op=dist.ReduceOp.MAX)
        s_ms = float(s_t.item())
        se = 2 if args.dtype == "bf16" else 4
        extras["strong_scaling"] = {
            "workload": args.strong_workload, "units": U, "units_per_rank": [(r * U) // world for r in range(world + 1)],
            "seq_len": sL, "d": sd, "w": sw_, "dtype": args.dtype, "ms_per_step": s_ms,
            "tokens_per_s": sB * sL / (s_ms / 1e3) if s_ms > 0 else None,
            "head_tokens_per_s": U * sL / (s_ms / 1e3) if s_ms > 0 else None,
            "hbm_frac_per_gpu": step_bytes_per_row(sd, se) * U * sL / world / (s_ms / 1e3) / 1e9 / hbm_peak
            if s_ms > 0 else None,
            "scaling": "strong", "timing": "compute only (slab resident on its GPU), CUDA events, max over ranks"}

    # (d) the other BASELINE configurations on one GPU, so the driver's record carries every
    # configs[] shape: C2b (Longformer-base, reading A14(b)) in both dtypes, C4 (configs[3],
    # dilation 2 and 4), the C5 sweep corners (configs[4]) -- ms per fwd + bwd step, the path,
    # and the step against its binding ceiling (HBM bytes of SURVEY.md §8(d) or tensor flops)
    if not args.no_extras and args.extra_steps > 0 and world == 1:
        others = {}
        for wl, odt in (("C2b", "bf16"), ("C2b", "f32"), ("C4d2", "bf16"), ("C4d4", "bf16"), ("C4d2", "f32"),
                        ("C5_w32", "bf16"), ("C5_w256", "bf16"), ("C5_small", "bf16"), ("C5_w32", "f32"),
                        ("C5_w256", "f32")):
            if wl == args.workload:
                continue
            oB, oH, oL, od, ow, odil = WORKLOADS[wl][:6]
            oe = 2 if odt == "bf16" else 4
            code = ft.FT_BF16 if odt == "bf16" else ft.FT_F32
            try:
                ms = quick_time(ft, torch, dev, (oB, oH, oL, od, ow, odil), odt, args.extra_steps, 3)
            except Exception as ex:
                others[f"{wl}/{odt}"] = {"error": f"{type(ex).__name__}: {ex}"[:200]}
                continue
            orows = oB * oH * oL
            hbm_f = step_bytes_per_row(od, oe) * orows / (ms / 1e3) / 1e9 / hbm_peak
            # band entries per row (exact), 12 d flops each for fwd + bwd; fp32 on the tensor cores
            # counts its 3 bf16 products
            n_i = float(window_sizes(oL, ow, odil).sum())
            fl = 12.0 * od * n_i * oB * oH * (3 if odt == "f32" else 1)
            ten_f = fl / (ms / 1e3) / (bf16_peak * 1e12)
            pth = dict(zip(("fwd", "bwd"), ("tc" if ft.plan(b_, oB, oH, oL, od, ow, odil, code)[0] == ft.PATH_TC
                                            else "simt" for b_ in (False, True))))
            others[f"{wl}/{odt}"] = {"shape": {"heads": oH, "seq_len": oL, "d": od, "w": ow, "dilation": odil},
                                     "ms_per_step": ms, "tokens_per_s": oB * oL / (ms / 1e3), "paths": pth,
                                     "hbm_frac": hbm_f, "tensor_frac": ten_f,
                                     "binding": "hbm" if hbm_f >= ten_f else "tensor"}
        extras["other_configs"] = others

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(shape, args.cpu_budget)

    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "tokens/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": elapsed_ms / args.steps,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None,
            "dtype": args.dtype, "data": "synthetic: U(-1,1) q/k/v/dout generated on device",
            **({"dtype_note": "fp32 storage and fp32 accuracy (north_star 1e-4 bound, parity-tested); the "
                              "tensor-core products are bf16 hi + lo splits, 3 per fp32 product, fp32 "
                              "accumulation (csrc/tc_band32.cu)"} if args.dtype == "f32" and path_b == ft.PATH_TC else {}),
            "config": cfg,
            "per_gpu_tokens_per_s": value / world,
            "paths": {"fwd": "tc" if path_f == ft.PATH_TC else "simt",
                      "bwd": "tc" if path_b == ft.PATH_TC else "simt"},
            "kernel_ms": {n: sum(x) / len(x) for n, x in kdur.items()},
            "kernel_timing": f"separate pass of {kpass} steps with an event after every launch "
                             "(serialised: no PDL overlap); the timed region has no per-launch events",
            "roofline": roof, "hbm_step": hbm_step, "ceilings": ceilings,
            "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": args.steps * (nf + nb),
            **({"e2e_nccl_scatter_gather": sg} if sg is not None else {}),
            **extras,
            "clocks": sampler.summary(),
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
