#!/usr/bin/env python
"""f2: the paper's index bijection on the B200 path, measured.

A session-structured stream (synth.workload.make_session_batch: every batch concentrates on one
topic's ids, scattered over the raw id space; the "local information" of P:206-208) is run
through the CUDA step (forward + backward + fused SGD, CUDA events) with three id maps:
  raw        -- the ids as they come,
  frequency  -- Alg. 2 lines 1-4 only (hot ids first, the rest in old order),
  community  -- Alg. 2 index graph + Louvain modularity communities,
the bijections built offline from K history batches and applied at run time in the key-build
kernel (ttemb_set_bijection).  Prints one JSON line per map: unique rows U and prefixes P
per step (the reuse Alg. 1 exploits), ms per step.

    python scripts/f2_measure.py [--tables 4] [--rows 2000000] [--batch 4096] [--hist 8]
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
from paper_conf_sc_wangwfmmd22_b200 import reorder  # noqa: E402
from synth import workload as W  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tables", type=int, default=4)
    ap.add_argument("--rows", type=int, default=2_000_000)
    ap.add_argument("--batch", type=int, default=4096)
    ap.add_argument("--hist", type=int, default=8)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--topics", type=int, default=8)
    ap.add_argument("--topic-frac", type=float, default=0.5)
    ap.add_argument("--topic-size", type=int, default=2048)
    ap.add_argument("--hot-ratio", type=float, default=0.0005)
    ap.add_argument("--window", type=int, default=32)
    a = ap.parse_args()
    f = W.near_cubic(a.rows)
    cfg = W.small_config([a.rows] * a.tables, [f] * a.tables, (4, 4, 4), 64, a.batch, 1, 1.05).replace(
        id_map="perm", name="f2-session")
    kw = dict(topics=a.topics, topic_frac=a.topic_frac, topic_size=a.topic_size)
    hist = [W.make_session_batch(cfg, step=s, seed=7, **kw) + (cfg.batch,) for s in range(a.hist)]
    t0 = time.time()
    maps = {"raw": None,
            "frequency": reorder.frequency_bijection(cfg.table_rows, hist, hot_ratio=a.hot_ratio)}
    t1 = time.time()
    maps["community"] = reorder.community_bijection(cfg.table_rows, hist, hot_ratio=a.hot_ratio, window=a.window)
    t2 = time.time()
    dev = torch.device("cuda", 0)
    B = cfg.batch
    pool = [W.make_session_batch(cfg, step=1000 + s, seed=9, **kw) for s in range(8)]
    dpool = [(torch.as_tensor(i, device=dev), torch.as_tensor(o, device=dev)) for i, o in pool]
    go = torch.as_tensor(W.make_grad_out(cfg, B, seed=9), device=dev)
    for name, bij in maps.items():
        emb = tt.TTEmbeddingBag.from_config(cfg, fused_update=True)
        emb.load_cores(W.make_cores(cfg, seed=9))
        if bij is not None:
            emb.set_bijection(torch.as_tensor(bij.view(np.int32), device=dev))
        out = torch.empty(B, cfg.num_tables, cfg.dim, device=dev)

        def step(i):
            di, do = dpool[i % len(dpool)]
            emb.forward(di, do, B, out=out)
            emb.backward(go, lr=0.01)
        for i in range(3):
            step(i)
        torch.cuda.synchronize()
        U = P = 0
        for i in range(len(dpool)):
            step(i)
            c = emb.counts()
            U += c["U"]
            P += c["P"]
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
        torch.cuda.synchronize()
        for i in range(a.steps):
            ev[i][0].record()
            step(i)
            ev[i][1].record()
        torch.cuda.synchronize()
        ms = sum(x.elapsed_time(y) for x, y in ev) / a.steps
        assert emb.check() == 0
        print(json.dumps({"map": name, "U_per_step": U / len(dpool), "P_per_step": P / len(dpool),
                          "ms_per_step": ms, "lookups_per_s": B * cfg.num_tables / (ms / 1e3),
                          "tables": a.tables, "rows": a.rows, "batch": B, "R": 64, "N": 64,
                          "build_s": {"frequency": round(t1 - t0, 2), "community": round(t2 - t1, 2)}.get(name)}),
              flush=True)


if __name__ == "__main__":
    main()
