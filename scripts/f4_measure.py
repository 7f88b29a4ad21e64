#!/usr/bin/env python
"""f4: the pipeline training system of PAPER §V measured in the Fig. 16 setup
(P:417): the largest table as a TT table in HBM (the tcgen05 path, fused SGD), the remaining
tables in host memory behind the parameter server, pre-fetch queue, embedding cache and gradient
queue (paper_conf_sc_wangwfmmd22_b200.hosttier).  Queue length 1 = "EL-Rec (Sequential)",
L > 1 = "EL-Rec (Pipeline)".  The model above the embeddings is the squared loss
1/2 |out - y|^2 (no MLPs: the GPU side is only the TT table, so the overlap the pipeline can find
is the server's work against the GPU step).  Prints one JSON line per queue length: samples/s
(wall clock over the timed steps, host work included: this is an end-to-end number).

    python scripts/f4_measure.py [--host-tables 8] [--host-rows 1000000] [--batch 4096]
"""
from __future__ import annotations

import argparse
import json
import os
import sys
import time

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_wangwfmmd22_b200 as tt  # noqa: E402
from paper_conf_sc_wangwfmmd22_b200.hosttier import HostTierEmbedding  # noqa: E402
from synth import workload as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--host-tables", type=int, default=8)
    ap.add_argument("--host-rows", type=int, default=1_000_000)
    ap.add_argument("--tt-rows", type=int, default=40_000_000)
    ap.add_argument("--batch", type=int, default=4096)
    ap.add_argument("--pooling", type=int, default=1)
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--queues", default="1,2,4,8")
    ap.add_argument("--no-cache", action="store_true", help="also time L>1 without the cache")
    a = ap.parse_args()
    dev = torch.device("cuda", 0)
    B, Lp = a.batch, a.pooling
    f = W.near_cubic(a.tt_rows)
    cfg = W.small_config([a.tt_rows], [f], (4, 4, 4), 64, B, Lp, 1.05).replace(name="f4-tt")
    emb = tt.TTEmbeddingBag.from_config(cfg, fused_update=True)
    emb.load_cores(W.make_cores(cfg, seed=3))
    hrows = [a.host_rows] * a.host_tables
    total = a.steps + a.warmup
    tt_batches = [tuple(torch.as_tensor(x, device=dev) for x in W.make_batch(cfg, step=k, seed=3)) for k in range(8)]
    host_batches = [W.make_host_batch(hrows, B, Lp, 1.05, step=k, seed=3) for k in range(total)]
    y_tt = torch.as_tensor(0.1 * W.make_grad_out(cfg, B, seed=3), device=dev)
    y_h = torch.as_tensor(0.1 * W.make_host_grad_out(a.host_tables, B, cfg.dim, seed=3), device=dev)
    W0 = W.make_host_weight(hrows, cfg.dim, seed=3)
    runs = [(int(q), True) for q in a.queues.split(",")]
    if a.no_cache:
        runs += [(int(q), False) for q in a.queues.split(",") if int(q) > 1]
    for L, cache in runs:
        ht = HostTierEmbedding(hrows, cfg.dim, B, a.host_tables * B * Lp, L, 0.01, use_cache=cache,
                               weight=W0)
        out_tt = torch.empty(B, 1, cfg.dim, device=dev)
        ht.start(lambda k: host_batches[k], total)
        t0 = None
        for k in range(total):
            if k == a.warmup:
                torch.cuda.synchronize()
                t0 = time.perf_counter()
            i, o = tt_batches[k % len(tt_batches)]
            emb.forward(i, o, B, out=out_tt)
            oh = ht.forward(k)
            emb.backward(out_tt - y_tt, lr=0.01)
            ht.backward((oh - y_h).contiguous())
            loss = ((oh - y_h) ** 2).sum()       # the step's result read back (a loss per step)
            loss.item()
        torch.cuda.synchronize()
        t1 = time.perf_counter()
        ht.finish()
        live, ovf = ht.cache_stats()
        host_ms = {k: round(1e3 * v / total, 3) for k, v in ht.times.items()}
        print(json.dumps({"queue_len": L, "cache": cache, "samples_per_s": a.steps * B / (t1 - t0),
                          "ms_per_step": 1e3 * (t1 - t0) / a.steps, "cache_live": live, "cache_overflow": ovf,
                          "cache_capacity": ht.capacity, "host_ms_per_step": host_ms, "host_tables": a.host_tables, "host_rows": a.host_rows,
                          "tt_rows": a.tt_rows, "batch": B, "pooling": Lp, "dim": cfg.dim}), flush=True)
        del ht


if __name__ == "__main__":
    main()
