#!/usr/bin/env python
"""How much does stash L2 residency matter?  Stage times of the c4 step at batch 4K / 8K / 16K
(P and dP stashes of ~30 / 60 / 120 MB against the 126 MB L2), normalised per unique prefix /
row.  Eager steps with per-stage CUDA events (ttemb_set_timing); the L2 is flushed between steps.

    python scripts/l2_probe.py
"""
import json
import os
import sys

import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_wangwfmmd22_b200 as tt  # noqa: E402
from synth import workload as W  # noqa: E402

dev = torch.device("cuda", 0)
base = W.config("c4")
flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
for B in (2048, 4096, 8192, 16384):
    cfg = base.replace(batch=B)
    emb = tt.TTEmbeddingBag.from_config(cfg, fused_update=True)
    emb.load_cores(W.make_cores(cfg, seed=0))
    pool = [W.make_batch(cfg, step=k, seed=0) for k in range(3)]
    dp = [(torch.as_tensor(i, device=dev), torch.as_tensor(o, device=dev)) for i, o in pool]
    go = torch.as_tensor(W.make_grad_out(cfg, B, seed=0), device=dev)
    out = torch.empty(B, cfg.num_tables, cfg.dim, device=dev)
    for k in range(3):
        emb.forward(*dp[k % 3], B, out=out)
        emb.backward(go, lr=0.01)
    torch.cuda.synchronize()
    emb.set_timing(True)
    n = 10
    for k in range(n):
        flush.fill_(k & 0xff)
        emb.forward(*dp[k % 3], B, out=out)
        emb.backward(go, lr=0.01)
    torch.cuda.synchronize()
    st = emb.stage_times()
    c = emb.counts()
    emb.set_timing(False)
    us = {k: v[0] / n * 1e3 for k, v in st.items() if v[1]}
    print(json.dumps({"batch": B, "U": c["U"], "P": c["P"], "NG": c["NG"],
                      "stash_MB": round(c["P"] * 4 * 256 * 4 / 1e6, 1),
                      "us": {k: round(v, 1) for k, v in us.items()},
                      "ns_per_prefix": {k: round(us[k] * 1e3 / c["P"], 2) for k in ("fwd_prefix", "bwd_prefix") if k in us},
                      "ns_per_row": {k: round(us[k] * 1e3 / c["U"], 2) for k in ("fwd_rows", "bwd_rows") if k in us}}),
          flush=True)
    del emb
