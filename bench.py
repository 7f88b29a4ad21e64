#!/usr/bin/env python
"""TT-EmbeddingBag fwd+bwd(+update) throughput on B200 (BASELINE.json metric).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c4] [--rank R]
                    [--impl ours|reference] [--opt sgd|adagrad] [--ids identity|perm]

One "step" = the whole hot path over one synthetic batch: index stage (sort /
unique / inverse / prefixes), prefix + row contractions, pooling, in-advance
aggregation, core-gradient contractions and the core update (fused when N=1;
NCCL all-reduce of the core gradients + update when N>1).  Prints ONE JSON line
on rank 0.  `--impl reference` times the CPU oracle (the tier's reference arm).
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

import numpy as np

if int(os.environ.get("WORLD_SIZE", "1")) > 1:
    # N > 1: the step graph interleaves NCCL kernels with ours; launch the main chain in plain
    # stream order there (PDL next to NCCL kernels was not validated on a multi-GPU box)
    os.environ.setdefault("TTEMB_NO_PDL", "1")

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from synth import workload as W  # noqa: E402

METRIC = "TT-EmbeddingBag fwd+bwd lookups/sec"
UNIT = "lookups/s"
HBM_PEAK_FALLBACK = 6650.0


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return (float(d.get("hbm_gbs", HBM_PEAK_FALLBACK)), float(d.get("sm_max_mhz", 1965.0)),
                float(d.get("bf16_tflops", 1590.0)), "measured")
    return HBM_PEAK_FALLBACK, 1965.0, 1590.0, "fallback"


def fp32_peak_tflops(sm_count: int, mhz: float) -> float:
    """FP32 FFMA peak: SMs x 128 FP32 lanes x 2 flop x clock."""
    return sm_count * 128 * 2 * mhz * 1e6 / 1e12


# ---------------------------------------------------------------------------
# clocks sampling during the timed region
# ---------------------------------------------------------------------------
class Clocks:
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_index: int):
        self.gpu = gpu_index
        self.rows = []
        self._stop = threading.Event()
        self._th = None

    def _run(self):
        while not self._stop.is_set():
            try:
                out = subprocess.run(["nvidia-smi", f"--id={self.gpu}", f"--query-gpu={self.Q}",
                                      "--format=csv,noheader,nounits"], capture_output=True,
                                     text=True, timeout=5).stdout.strip()
                if out:
                    self.rows.append([x.strip() for x in out.split(",")])
            except Exception:
                pass
            self._stop.wait(0.05)

    def __enter__(self):
        self._th = threading.Thread(target=self._run, daemon=True)
        self._th.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self._th:
            self._th.join(timeout=10)

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"], "samples": 0}
        sm = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = set()
        for r in self.rows:
            for n, v in zip(names, r[5:9]):
                if v.strip().lower() == "active":
                    reasons.add(n)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(self.rows)}


# ---------------------------------------------------------------------------
# algorithmic work
# ---------------------------------------------------------------------------
def step_work(cfg, B, nnz, counts, touched, opt, tc):
    """(tensor_flops, alu_flops, bytes) of one step: the rank-R prefix contractions (fwd a5 + bwd
    a10, 3 x 2 n1 n2 R^2 per unique prefix) on tcgen05 when `tc`, the row contractions (a6, a9:
    3 x 2 N R per unique row) on FFMA; bytes per SURVEY 8(d)."""
    n1, n2, n3 = cfg.col_factors
    R, N, T = cfg.rank, cfg.dim, cfg.num_tables
    U, P = counts["U"], counts["P"]
    nd = touched.get("dense_rows", 0)                  # hybrid: plain rows (no TT arithmetic)
    pf = 3 * 2 * n1 * n2 * R * R * P
    rf = 3 * 2 * N * R * (U - nd)
    slice_bytes = 4 * (touched["c1"] * n1 * R + touched["c2"] * R * n2 * R + touched["c3"] * R * n3
                       + nd * N)
    passes = 3 if opt == "sgd" else 5                  # fwd read, bwd read, update write (+ state r/w)
    bytes_ = 8 * nnz + 8 * (T * B + 1) + 2 * 4 * N * T * B + passes * slice_bytes
    return (pf if tc else 0), rf + (0 if tc else pf), bytes_


def stage_work(name, cfg, B, nnz, counts, tc=False):
    """Algorithmic work of one launch of a stage: (tensor_flops, alu_flops, bytes).
    tensor_flops are the rank-R prefix contractions when they run on tcgen05 (3xTF32), alu_flops
    the FP32 FFMA work (row contractions; the prefix contractions on the FFMA path), bytes the
    algorithmic HBM bytes (touched slices, ids, out / grad_out; intermediates a
    fused design keeps on chip are not counted)."""
    n1, n2, n3 = cfg.col_factors
    R, N, T = cfg.rank, cfg.dim, cfg.num_tables
    U, P, NG = counts["U"], counts["P"], counts["NG"]
    c2 = 4 * NG * R * n2 * R
    pf = 2 * n1 * n2 * R * R * P

    def split(f):
        return (f, 0) if tc else (0, f)
    if name == "fwd_prefix":                      # a5 (+ a6 when fused)
        return (*split(pf), c2 + 4 * P * n1 * R)
    if name == "fwd_rows":
        return 0, 2 * N * R * U, 4 * U * N
    if name == "fwd_fused":                       # a5 + a6 (+ a7 for one-id bags)
        return (*split(pf), 2 * N * R * U, c2 + 4 * P * n1 * R + 4 * N * T * B)
    if name == "bwd_prefix":                      # a10 - a12
        return (*split(2 * pf), 2 * c2 + 4 * P * n1 * R)
    if name == "bwd_rows":
        return 0, 4 * N * R * U, 4 * U * N
    if name == "bwd_fused":                       # a9 - a12 (prefix recomputed on chip)
        return (*split(3 * pf), 4 * N * R * U, 2 * c2 + 4 * P * n1 * R + 4 * U * N)
    if name == "pool":
        return 0, 0, 4 * N * T * B + 4 * N * nnz + 4 * nnz + 8 * (T * B + 1)
    if name == "agg":
        return 0, 0, 4 * N * nnz + 8 * nnz + 4 * N * U
    if name == "sort_pass":
        return 0, 0, 16 * nnz
    return 0, 0, 0


def plan_work(cfg, idx, off, B):
    """Algorithmic FLOPs of one batch from its unique rows / prefixes (numpy)."""
    n1, n2, n3 = cfg.col_factors
    R, N, T = cfg.rank, cfg.dim, cfg.num_tables
    tab = np.repeat(np.arange(T * B), np.diff(off)) // B
    U = P = 0
    for t in range(T):
        ids = np.unique(np.asarray(idx)[tab == t])
        if getattr(cfg, "dense", ()) and cfg.dense[t]:
            continue
        m3 = cfg.row_factors[t][2]
        U += len(ids)
        P += len(np.unique(ids // m3))
    return 3 * 2 * n1 * n2 * R * R * P + 3 * 2 * N * R * U


def scaling_cap(cfg, world, args):
    """SURVEY 8(e) work model: per-GPU dedup shrinks slower than 1/G, so with a fixed global
    batch (strong scaling) the best possible efficiency is W(1) / (G max_g W_g) with W the
    algorithmic FLOPs of a batch; with a fixed per-GPU batch (weak scaling) the work per GPU does
    not change (cap 1, minus the gradient exchange)."""
    if world == 1 or args.scaling == "weak":
        return {"kind": args.scaling, "cap": 1.0, "model": "per-GPU work fixed"}
    gi, goff = W.make_batch(cfg, step=0, seed=args.seed)
    w1 = plan_work(cfg, gi, goff, cfg.batch)
    shards = [W.shard_batch(gi, goff, cfg.num_tables, cfg.batch, r, world) for r in range(world)]
    wg = max(plan_work(cfg, i, o, b) for i, o, b in shards)
    return {"kind": "strong", "cap": w1 / (world * wg), "model": "alg FLOPs of the global batch / (G x max shard)",
            "gflop_global": w1 / 1e9, "gflop_max_shard": wg / 1e9}


def kernel_roofline(name, work, per_launch_ms, hbm_peak, tensor_peak, alu_peak):
    """The binding roofline of one launch: the largest of (tensor flops at the 3xTF32 peak, FFMA
    flops at the FP32 peak, algorithmic bytes at the HBM peak); achieved = that quantity per
    measured launch time, frac = floor time / measured time."""
    tf, af, by = work
    t = {"tensor": tf / (tensor_peak * 1e12), "alu": af / (alu_peak * 1e12), "hbm": by / (hbm_peak * 1e9)}
    bound = max(t, key=t.get)
    sec = per_launch_ms / 1e3
    if bound == "hbm":
        ach, peak, unit = by / sec / 1e9, hbm_peak, "GB/s"
    elif bound == "tensor":
        ach, peak, unit = tf / sec / 1e12, tensor_peak, "TFLOP/s"
    else:
        ach, peak, unit = af / sec / 1e12, alu_peak, "TFLOP/s"
    return {"bound": bound, "kernel": name, "achieved": ach, "peak": peak, "unit": unit, "frac": ach / peak,
            "floors_us": {k: round(v * 1e6, 2) for k, v in t.items()}, "measured_us": round(per_launch_ms * 1e3, 2),
            "work": {"tensor_gflop": tf / 1e9, "alu_gflop": af / 1e9, "alg_mb": by / 1e6}}


# ---------------------------------------------------------------------------
# reference arm: the CPU oracle as it stands
# ---------------------------------------------------------------------------
def oracle_step(orc, cfg, cores, idx, off, b, go, lr, opt):
    orc.forward(cores, idx, off, b)
    g = orc.backward(cores, idx, off, b, go)
    new = []
    for t, c in enumerate(cores):
        new.append(tuple(orc.update(opt, lr, c[k], g[t][k])[0] for k in range(3)))
    return new


def sub_batch(idx, off, T, B, b):
    """The first b samples of every table of a (T, B) batch."""
    parts, lens = [], []
    for t in range(T):
        s, e = off[t * B], off[t * B + b]
        parts.append(idx[s:e])
        lens.append(np.diff(off[t * B:t * B + b + 1]))
    lens = np.concatenate(lens)
    o = np.zeros(T * b + 1, np.int64)
    np.cumsum(lens, out=o[1:])
    return np.concatenate(parts), o


def calibrate_sample(orc, cfg, cores, idx, off, B, go, lr, opt, target_s):
    b = max(1, min(B, 64))
    while True:
        si, so = sub_batch(idx, off, cfg.num_tables, B, b)
        t0 = time.perf_counter()
        oracle_step(orc, cfg, cores, si, so, b, go[:b], lr, opt)
        dt = time.perf_counter() - t0
        if dt >= 0.25 * target_s or b >= B:
            break
        b = min(B, b * 4)
    scale = target_s / max(dt, 1e-6)
    return max(1, min(B, int(b * scale)))


def cpu_baseline(cfg, cores, idx, off, B, go, lr, opt, target_s=15.0):
    import oracle
    orc = oracle.Oracle.from_config(cfg)
    b = calibrate_sample(orc, cfg, cores, idx, off, B, go, lr, opt, target_s)
    si, so = sub_batch(idx, off, cfg.num_tables, B, b)
    t0 = time.perf_counter()
    oracle_step(orc, cfg, cores, si, so, b, go[:b], lr, opt)
    dt = time.perf_counter() - t0
    look = int(so[-1])
    return {"value": look / dt, "unit": UNIT, "cores": oracle.Oracle.num_threads(), "kind": "oracle",
            "sample": f"first {b} of {B} samples of every table of step-0 batch ({look} lookups), "
                      f"fp64 oracle fwd+bwd+{opt} update, {dt:.1f} s wall"}


def run_reference(args, cfg, rank, world):
    if rank != 0:
        return
    # torchrun pins OMP_NUM_THREADS=1 per rank; rank 0 runs the oracle alone on the host cores
    os.environ["OMP_NUM_THREADS"] = str(os.cpu_count() or 1)
    import oracle
    B = cfg.batch if args.scaling == "weak" else cfg.batch // world
    cores = W.make_cores(cfg, seed=args.seed)
    idx, off = W.make_batch(cfg, step=0, seed=args.seed, batch=B)
    go = W.make_grad_out(cfg, B, step=0, seed=args.seed)
    orc = oracle.Oracle.from_config(cfg)
    budget = 150.0 / max(1, args.steps + args.warmup)
    b = calibrate_sample(orc, cfg, cores, idx, off, B, go, args.lr, args.opt, budget)
    si, so = sub_batch(idx, off, cfg.num_tables, B, b)
    for _ in range(args.warmup):
        oracle_step(orc, cfg, cores, si, so, b, go[:b], args.lr, args.opt)
    t0 = time.perf_counter()
    for _ in range(args.steps):
        cores = oracle_step(orc, cfg, cores, si, so, b, go[:b], args.lr, args.opt)
    dt = time.perf_counter() - t0
    look = int(so[-1]) * args.steps
    val = look / dt
    line = {"metric": METRIC, "value": val, "unit": UNIT, "impl": "reference", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * dt / args.steps,
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f64",
            "data": "synthetic", "config": workload_config(cfg, B, world, args),
            "cpu_baseline": {"value": val, "unit": UNIT, "cores": oracle.Oracle.num_threads(),
                             "kind": "oracle",
                             "sample": f"first {b} of {B} samples of every table per step "
                                       f"({int(so[-1])} lookups), fp64 oracle fwd+bwd+{args.opt} update"},
            "e2e": {"value": val, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_paper(args, cfg, rank, world):
    """--impl paper: the paper's own GPU design (Alg. 1 reuse buffer + cuBLAS batched GEMMs,
    aggregation by index_add; comparators/paper_design.py) on the same workload and GPU,
    timed like our arm (device events, L2 flushed between steps).  SURVEY.md 8(f1)."""
    import torch
    from comparators.paper_design import PaperDesignTT
    torch.backends.cuda.matmul.allow_tf32 = False
    if world > 1 and rank != 0:
        return
    dev = torch.device("cuda", int(os.environ.get("LOCAL_RANK", "0")))
    torch.cuda.set_device(dev)
    B = cfg.batch
    pool = []
    for i in range(min(args.pool, 2)):
        idx, off = W.make_batch(cfg, step=i, seed=args.seed, batch=B)
        go = W.make_grad_out(cfg, B, step=i, seed=args.seed)
        pool.append((torch.as_tensor(idx, device=dev), torch.as_tensor(off, device=dev),
                     torch.as_tensor(go, device=dev)))
    m = PaperDesignTT(cfg.table_rows, cfg.row_factors, cfg.col_factors, cfg.rank, dev)
    m.load_cores(W.make_cores(cfg, seed=args.seed))
    offs_host = [p[1].cpu() for p in pool]
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)

    def step(i):
        di, do, dg = pool[i % len(pool)]
        m.forward(di, offs_host[i % len(pool)], B)
        m.backward(dg)
        m.update_sgd(args.lr)

    for i in range(args.warmup):
        step(i)
    torch.cuda.synchronize()
    stream = torch.cuda.current_stream()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    with Clocks(dev.index) as clk:
        for i in range(args.steps):
            flush.fill_(i & 0xff)
            ev[i][0].record(stream)
            step(i)
            ev[i][1].record(stream)
        torch.cuda.synchronize()
    t_ms = sum(a.elapsed_time(b) for a, b in ev)
    look = sum(int(p[0].shape[0]) for p in pool) / len(pool)
    val = look * args.steps / (t_ms / 1e3)
    line = {"metric": METRIC, "value": val, "unit": UNIT, "impl": "paper-design", "n_gpus": 1,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": t_ms / args.steps,
            "higher_is_better": True, "scaling": args.scaling, "vs_baseline": None, "dtype": "f32",
            "data": "synthetic", "config": workload_config(cfg, B, 1, args),
            "design": "Alg. 1 reuse buffer (torch.unique owners) + cuBLAS batched GEMM stages, index_add "
                      "aggregation / pooling / core-gradient reduction, unfused SGD (P:178-196, P:346)",
            "clocks": clk.summary()}
    line["config"]["update"] = "unfused"
    print(json.dumps(line), flush=True)


def workload_config(cfg, B, world, args):
    return {"workload": cfg.name, "tables": cfg.num_tables, "max_rows": max(cfg.table_rows),
            "dim": cfg.dim, "col_factors": list(cfg.col_factors), "tt_rank": cfg.rank,
            "batch_per_gpu": B, "global_batch": B * world, "pooling": cfg.pooling,
            "ids": f"zipf{cfg.zipf_s}-{cfg.id_map}" if cfg.zipf_s else f"uniform-{cfg.id_map}",
            "optimizer": args.opt,
            "update": ("fused" if world == 1 and not getattr(args, "unfused", False)
                       else ("bucketed all-reduce + update" if getattr(args, "grad_sync", "allreduce") == "allreduce"
                             else "reduce-scatter + sharded update + all-gather") if world > 1 else "unfused"),
            "parallelism": f"dp{world}", "l2": "flushed between timed steps (untimed 512 MiB write)",
            **({"bijection": f"frequency order (Alg. 2 l.1-4), {args.bijection} history batches"}
               if getattr(args, "bijection", 0) else {}),
            **({"ablation": [k for k in ("no_reuse", "no_agg", "unfused") if getattr(args, k, False)]}
               if any(getattr(args, k, False) for k in ("no_reuse", "no_agg", "unfused")) else {})}


# ---------------------------------------------------------------------------
# our arm
# ---------------------------------------------------------------------------
def kernels_per_step(emb_ctx, world, fused=True, cfg=None, fused_update=None):
    """Our kernel launches per step (cudaMemsetAsync excluded), matching the ncu launch list.
    tcgen05 path: index stage = build_keys + hist_scan + kp radix passes + plan scan + the
    plan-dependent zeroing (zero_rows, dp_zero2); forward = gather-table prep + prefix GEMM + rows
    + two pool launches (one-id copy / bag sums; the one not needed exits); backward = agg + rows_bwd + prefix GEMM bwd + one update (k_update_zero
    when fused, k_update after the all-reduce otherwise).  FFMA path: build_keys + hist_scan + kp
    passes + plan scan + zero_rows; group fwd + pool; agg + group bwd + dc1 + update."""
    kp, _ = emb_ctx
    if fused:
        return (1 + 1 + kp + 1 + 2) + 5 + 4    # fwd = prep + prefix + rows + two pool launches
    return (1 + 1 + kp + 1 + 1) + 3 + 4


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=200)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--config", default="c4")
    ap.add_argument("--rank", type=int, default=None, help="TT rank for c5 (32/64/128)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference", "paper"],
                    help="reference = the CPU oracle; paper = the paper's design in torch/cuBLAS")
    ap.add_argument("--opt", default="sgd", choices=["sgd", "adagrad"])
    ap.add_argument("--ids", default="identity", choices=["identity", "perm"])
    ap.add_argument("--scaling", default=None, choices=["weak", "strong"])
    ap.add_argument("--pool", type=int, default=4, help="distinct pre-generated batches")
    ap.add_argument("--lr", type=float, default=0.01)
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--e2e-depth", type=int, default=2, help="HostStepPipeline staging slots for the e2e leg")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--stages", action="store_true", help="print per-stage times to stderr")
    ap.add_argument("--fp32-cores", action="store_true", help="force the FFMA contraction path (no tcgen05)")
    ap.add_argument("--no-reuse", action="store_true",
                    help="ablation: no batch-level prefix reuse (TTEMB_NO_PREFIX_REUSE, P:419)")
    ap.add_argument("--no-agg", action="store_true",
                    help="ablation: no row dedup / in-advance gradient aggregation (TTEMB_NO_AGGREGATION, P:416)")
    ap.add_argument("--unfused", action="store_true",
                    help="ablation: backward writes dense core grads, separate update (P:421)")
    ap.add_argument("--bijection", type=int, default=0, metavar="K",
                    help="f2: frequency-ordering index bijection (Alg. 2 l.1-4) built offline from K "
                         "history batches of the stream, applied at run time (P:269)")
    ap.add_argument("--hybrid", action="store_true",
                    help="f3: hybrid placement -- tables with <= 1M rows stay dense (P:310)")
    ap.add_argument("--no-pipeline", dest="pipeline", action="store_false",
                    help="no cross-step pipelining of the next batch's index stage")
    ap.add_argument("--no-graph", dest="graph", action="store_false",
                    help="launch every step eagerly instead of replaying a captured CUDA graph")
    ap.add_argument("--grad-sync", default="allreduce", choices=["allreduce", "rs_ag"],
                    help="N > 1: bucketed all-reduce overlapped with the backward, or reduce-scatter -> "
                         "sharded update -> all-gather (SURVEY 8(e))")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    cfg = W.config(args.config, args.rank) if args.config == "c5" else W.config(args.config)
    cfg = cfg.replace(id_map=args.ids)
    if args.hybrid:
        cfg = W.hybrid(cfg)
    if args.scaling is None:
        args.scaling = "strong" if args.config == "c5" else "weak"

    if args.impl == "reference":
        # rank 0 alone times the oracle; no process group (and no torch import, whose OpenMP
        # runtime would pin the oracle to torchrun's OMP_NUM_THREADS=1)
        run_reference(args, cfg, rank, world)
        return
    if args.impl == "paper":
        run_paper(args, cfg, rank, world)
        return

    import torch
    import torch.distributed as dist
    import paper_conf_sc_wangwfmmd22_b200 as tt
    from paper_conf_sc_wangwfmmd22_b200 import parallel

    # one rank per GPU; on a box with fewer GPUs than ranks (a functional check of the N > 1
    # path only) ranks share devices and the all-reduce falls back to gloo
    ndev = torch.cuda.device_count()
    shared = world > ndev
    local_rank = local_rank % ndev
    torch.cuda.set_device(local_rank)
    dev = torch.device("cuda", local_rank)
    if world > 1:
        if shared:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=dev)
    B = cfg.batch if args.scaling == "weak" else cfg.batch // world
    fused = world == 1 and not args.unfused

    # ---- inputs: a pool of batches resident in HBM ----
    pool = []
    for i in range(args.pool):
        if args.scaling == "weak":
            idx, off = W.make_batch(cfg, step=i, seed=args.seed + 1000 * rank, batch=B)
            go = W.make_grad_out(cfg, B, step=i, seed=args.seed + 1000 * rank)
        else:
            gi, goff = W.make_batch(cfg, step=i, seed=args.seed)
            idx, off, _ = W.shard_batch(gi, goff, cfg.num_tables, cfg.batch, rank, world)
            go = W.make_grad_out(cfg, cfg.batch, step=i, seed=args.seed)[rank * B:(rank + 1) * B].copy()
        pool.append((idx, off, go))
    max_nnz = max(len(p[0]) for p in pool)
    emb = tt.TTEmbeddingBag(cfg.table_rows, cfg.row_factors, cfg.col_factors, cfg.rank, B, max_nnz,
                            dense=cfg.dense,
                            optimizer=args.opt, fused_update=fused, device=local_rank,
                            fp32_cores=args.fp32_cores, prefix_reuse=not args.no_reuse,
                            aggregation=not args.no_agg)
    cores = W.make_cores(cfg, seed=args.seed)
    emb.load_cores(cores)
    bij_t = None
    if args.bijection:
        from paper_conf_sc_wangwfmmd22_b200 import reorder
        hist = (W.make_batch(cfg, step=10_000 + k, seed=args.seed + 1000 * rank, batch=B) + (B,)
                for k in range(args.bijection))
        bij_t = torch.as_tensor(reorder.frequency_bijection(cfg.table_rows, hist).view(np.int32), device=dev)
        emb.set_bijection(bij_t)
    dpool = [(torch.as_tensor(i, device=dev), torch.as_tensor(o, device=dev), torch.as_tensor(g, device=dev))
             for i, o, g in pool]
    out = torch.empty(B, cfg.num_tables, cfg.dim, device=dev)
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream()

    sync = parallel.GradSync(emb, mode=args.grad_sync) if not fused else None

    def step(i):
        di, do, dg = dpool[i % len(dpool)]
        emb.forward(di, do, B, out=out)
        emb.backward(dg, lr=args.lr)
        if sync is not None:
            sync.exchange_and_update(args.lr)

    # ---- cross-step pipelining (default): the index stage of batch g+1 (ttemb_plan_batch, reads no
    #      parameters) runs on a side stream while batch g's forward compute + backward + update run;
    #      two handles on the same cores / grads alternate so each keeps its own plan.  Every timed
    #      step = one batch's compute + the next batch's index stage, joined at the step's end. ----
    pipe = args.pipeline and len(dpool) % 2 == 0
    if pipe:
        embs = [emb, emb.sibling()]
        hsync = [sync, parallel.GradSync(embs[1], mode=args.grad_sync, comm_stream=sync.comm)] \
            if sync is not None else None
        side = torch.cuda.Stream(device=dev)
        ev_go = [torch.cuda.Event() for _ in range(len(dpool))]
        ev_planned = [torch.cuda.Event() for _ in range(len(dpool))]
        gstate = {"g": 0}

        def pstep(g):
            cur = torch.cuda.current_stream()
            h, nh = embs[g % 2], embs[(g + 1) % 2]
            _, _, dg = dpool[g % len(dpool)]
            ni, no, _ = dpool[(g + 1) % len(dpool)]
            e_go, e_pl = ev_go[g % len(dpool)], ev_planned[g % len(dpool)]
            e_go.record(cur)                 # nh's previous step (g-1) is queued before this point
            h.forward_planned(out)
            side.wait_event(e_go)
            nh.plan_batch(ni, no, B, stream=side)
            e_pl.record(side)
            h.backward(dg, lr=args.lr)
            if sync is not None:
                hsync[g % 2].exchange_and_update(args.lr)
            cur.wait_event(e_pl)

        embs[0].plan_batch(dpool[0][0], dpool[0][1], B)

        def step_pipe(_i):
            pstep(gstate["g"])
            gstate["g"] += 1
    for i in range(args.warmup):
        step_pipe(i) if pipe else step(i)
    torch.cuda.synchronize()
    assert emb.check() == 0, "device-side input error"

    # ---- optional CUDA graphs: one captured step per pool batch (same kernels, no launch gaps) ----
    graphs = None
    # CUDA graphs: NCCL collectives are capturable; the gloo fallback (ranks sharing a GPU) is not
    if args.graph and (world == 1 or not shared):
        torch.cuda.synchronize()
        graphs = []
        g0 = gstate["g"] if pipe else 0
        for i in range(len(dpool)):
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g):
                pstep(g0 + i) if pipe else step(i)
            graphs.append(g)
        for i in range(len(graphs)):
            graphs[i].replay()
        torch.cuda.synchronize()
        assert emb.check() == 0, "device-side input error (graph replay)"

    def run(i):
        if graphs is not None:
            graphs[i % len(graphs)].replay()
        elif pipe:
            step_pipe(i)
        else:
            step(i)

    # ---- timed region (device events per step; L2 flushed between steps, untimed) ----
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    with Clocks(local_rank) as clk:
        for i in range(args.steps):
            flush.fill_(i & 0xff)
            ev[i][0].record(stream)
            run(i)
            ev[i][1].record(stream)
        torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    t_ms = sum(a.elapsed_time(b) for a, b in ev)
    t_max = torch.tensor([t_ms], dtype=torch.float64, device=dev)
    if world > 1:
        dist.all_reduce(t_max, op=dist.ReduceOp.MAX)
    t_ms = float(t_max.item())
    look_step = sum(int(p[0].shape[0]) for p in pool) / len(pool)
    value = world * look_step * args.steps / (t_ms / 1e3)

    # ---- per-stage breakdown: a separate eager pass with CUDA events around every stage on the
    #      launching stream (kept out of the timed region so the events do not perturb it) ----
    emb.set_timing(True)
    emb.stage_times()   # reset
    for i in range(args.steps):
        flush.fill_(i & 0xff)
        step(i)
    torch.cuda.synchronize()
    stages = emb.stage_times()
    emb.set_timing(False)
    stage_total_ms = sum(v[0] for v in stages.values())

    # ---- counts of the last step for the roofline ----
    counts = emb.counts()
    plan = emb.plan()
    last = (args.steps - 1) % len(pool)
    nnz_last = len(pool[last][0])
    pt = plan["pfx_t"].cpu().numpy().astype(np.int64)
    pi1 = plan["pfx_i1"].cpu().numpy().astype(np.int64)
    rp = plan["row_pfx"].cpu().numpy().astype(np.int64) & 0xFFFFFFFF
    tt_row = rp != 0xFFFFFFFF                       # hybrid: dense-table rows have no prefix
    ri3 = plan["row_i3"].cpu().numpy().astype(np.int64)[tt_row]
    rt = pt[rp[tt_row]]
    touched = {"c1": len(np.unique(pt * (1 << 32) + pi1)), "c2": counts["NG"],
               "c3": len(np.unique(rt * (1 << 32) + ri3)), "dense_rows": int((~tt_row).sum())}
    hbm_peak, sm_max_mhz, bf16_peak, peak_kind = load_peaks()
    on_tc = tc_path(cfg, args)
    sm_count = torch.cuda.get_device_properties(dev).multi_processor_count
    alu_peak = fp32_peak_tflops(sm_count, sm_max_mhz)
    tflops, aflops, bytes_ = step_work(cfg, B, nnz_last, counts, touched, args.opt, on_tc)
    tensor_peak = bf16_peak / 2.0 / 3.0          # 3xTF32: 3 TF32 MMAs per fp32 product, TF32 = bf16 / 2
    ms_step = t_ms / args.steps
    # dominant kernel (stage) of the eager breakdown; its binding roofline
    dom = max(stages.items(), key=lambda kv: kv[1][0])
    dname, (dms, dn) = dom
    per_launch_ms = dms / max(dn, 1)
    roof = kernel_roofline(dname, stage_work(dname, cfg, B, nnz_last, counts, tc=on_tc), per_launch_ms,
                           hbm_peak, tensor_peak, alu_peak)
    roof["peak_source"] = {"hbm": f"{peak_kind} copy bandwidth (MEASURED_PEAKS.json hbm_gbs)",
                           "tensor": f"{peak_kind} bf16 {bf16_peak:.0f} TFLOP/s x 1/2 (tf32) x 1/3 (3xTF32)",
                           "alu": f"derived: {sm_count} SM x 128 FP32 FMA/clk x 2 x {sm_max_mhz:.0f} MHz"}[roof["bound"]]
    roof["share_of_step"] = dms / max(stage_total_ms, 1e-9)
    roof["traffic"] = None
    tr_path = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tr_path):      # DRAM bytes per launch from a committed ncu --set full capture of THIS config
        tr = json.load(open(tr_path))
        key = f"{cfg.name}-r{cfg.rank}/{dname}"
        if key in tr.get("dram_bytes_per_launch", {}):
            roof["traffic"] = tr["dram_bytes_per_launch"][key]
            roof["traffic_source"] = tr.get("source")
    t_tc = tflops / (tensor_peak * 1e12) * 1e3
    t_alu = aflops / (alu_peak * 1e12) * 1e3
    t_hbm = bytes_ / (hbm_peak * 1e9) * 1e3
    t_cmp = t_tc + t_alu                           # tensor and FFMA work counted serially
    step_roof = {"alg_gflop_tensor": tflops / 1e9, "alg_gflop_alu": aflops / 1e9, "alg_mb": bytes_ / 1e6,
                 "t_tensor_ms": t_tc, "t_alu_ms": t_alu, "t_hbm_ms": t_hbm,
                 "frac_hbm_roofline": t_hbm / ms_step, "frac_binding_roofline": max(t_cmp, t_hbm) / ms_step,
                 "binding": "hbm" if t_hbm >= t_cmp else ("tensor+alu" if t_tc and t_alu else "alu"),
                 "U": counts["U"], "P": counts["P"],
                 "NG": counts["NG"], "touched_slices": touched}

    # ---- end-to-end from pinned host memory: every step copies its inputs in and its pooled ----
    # ---- output back; HostStepPipeline overlaps step k+1's input copy and step k-1's output ----
    # ---- copy with step k's kernels (two staging slots)                                      ----
    e2e = None
    if not args.no_e2e and world == 1:
        hpool = [(torch.as_tensor(i).pin_memory(), torch.as_tensor(o).pin_memory(),
                  torch.as_tensor(g).pin_memory()) for i, o, g in pool]
        depth = args.e2e_depth
        houts = [torch.empty(B, cfg.num_tables, cfg.dim).pin_memory() for _ in range(depth)]
        pipe = tt.HostStepPipeline(emb, max(p[0].numel() for p in hpool), B, depth=depth)

        def hstep(i):
            hi, ho, hg = hpool[i % len(hpool)]
            return pipe.step(hi, ho, hg, houts[i % depth], lr=args.lr)

        with torch.cuda.stream(stream):
            for i in range(args.warmup):
                hstep(i)
            torch.cuda.synchronize()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(pipe.h2d)                    # before the first input copy
            last = 0
            for i in range(args.steps):
                flush.fill_(i & 0xff)
                last = hstep(i)
            e1.record(pipe.d2h)                    # after the last output copy
            pipe.wait(last)
            torch.cuda.synchronize()
        te = e0.elapsed_time(e1)
        h2d = sum(p[0].size * 8 + p[1].size * 8 + p[2].size * 4 for p in pool) / len(pool)
        e2e = {"value": look_step * args.steps / (te / 1e3), "unit": UNIT, "h2d_bytes_per_step": int(h2d),
               "d2h_bytes_per_step": int(houts[0].numel() * 4), "ms_per_step": te / args.steps,
               "path": "HostStepPipeline: pinned host ids / offsets / grad_out -> device, "
                       "ttemb_forward + ttemb_backward, pooled output -> pinned host; copies of "
                       f"neighbouring steps overlapped with compute ({depth} staging slots)"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        idx0, off0, go0 = pool[0]
        cpu = cpu_baseline(cfg, cores, idx0, off0, B, go0, args.lr, args.opt)

    if args.stages and rank == 0:
        for k, (ms, n) in sorted(stages.items(), key=lambda kv: -kv[1][0]):
            if n:
                print(f"  {k:12s} {ms / args.steps * 1e3:9.1f} us/step  ({n} launches)", file=sys.stderr)

    if rank == 0:
        line = {"metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True,
                "scaling": args.scaling, "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": workload_config(cfg, B, world, args), "roofline": roof,
                "step_roofline": step_roof, "cpu_baseline": cpu, "e2e": e2e,
                "gpu_launches": kernels_per_step(emb_passes(emb), world, fused=tc_path(cfg, args),
                                                 fused_update=fused) * args.steps,
                "graph": bool(graphs is not None),
                **({"scaling_cap": scaling_cap(cfg, world, args)} if world > 1 else {}),
                "pipeline": "next batch's index stage on a side stream" if pipe else None,
                "clocks": clk.summary(),
                "stages_us_per_step": {k: round(v[0] / args.steps * 1e3, 2) for k, v in stages.items() if v[1]}}
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def tc_path(cfg, args):
    """The tcgen05 path (R = 64, n2 R <= 256, n3 in {4, 8}, n1 a power of two <= 8)."""
    n1, n2, n3 = cfg.col_factors
    # ranks 16..31 / 33..63 run zero-padded to 32 / 64 (R28); 32, 64, 128 natively
    R = 32 if 16 <= cfg.rank <= 32 else 64 if 32 < cfg.rank <= 64 else cfg.rank
    return (not args.fp32_cores) and R in (32, 64, 128) and n3 in (4, 8) and n1 in (1, 2, 4, 8) \
        and n1 * n2 <= 16 and n2 * R <= (512 if R == 128 else 256)


def emb_passes(emb):
    keys = sum(int(f[0]) * int(f[1]) * int(f[2]) for f in emb.row_factors)   # group-major plan keys
    kp = max(1, (max(keys - 1, 0).bit_length() + 7) // 8)
    gb = sum(f[1] for f in emb.row_factors)
    gp = max(1, (max(gb - 1, 0).bit_length() + 7) // 8)
    return kp, gp


if __name__ == "__main__":
    main()
