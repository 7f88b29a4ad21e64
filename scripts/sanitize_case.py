"""One small forward + backward (+ update) through the C ABI, for compute-sanitizer runs:
    compute-sanitizer --tool memcheck python scripts/sanitize_case.py <case>"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sc_wangwfmmd22_b200 as tt  # noqa: E402
from synth import workload as W  # noqa: E402

CASES = {
    "c1": (lambda: W.config("c1"), {}),
    "c2-b256": (lambda: W.config("c2"), dict(batch=256)),
    "tc-r64": (lambda: W.small_config([20000, 300], [(28, 28, 26), (7, 7, 7)], (4, 4, 4), 64, 96, 2, 1.05), {}),
    "ffma-split": (lambda: W.small_config([200000], [(2000, 10, 10)], (2, 2, 4), 16, 512, 2, 0.9), dict(fp32=True)),
    "tc-r32": (lambda: W.small_config([20000, 300], [(28, 28, 26), (7, 7, 7)], (4, 4, 4), 32, 96, 2, 1.05), {}),
    "tc-r128": (lambda: W.small_config([20000, 300], [(28, 28, 26), (7, 7, 7)], (4, 4, 8), 128, 64, 2, 1.05), {}),
}
name = sys.argv[1]
if name == "hosttier":      # f4: host-memory tier kernels (cache sync / pool / grad / tick / update-push)
    from paper_conf_sc_wangwfmmd22_b200.hosttier import HostTierEmbedding
    rows, B, L = [300, 50, 800], 32, 3
    batches = [W.make_host_batch(rows, B, 3, 1.05, step=k, seed=1) for k in range(6)]
    ht = HostTierEmbedding(rows, 16, B, len(rows) * B * 3, L, 0.05, threaded=False,
                           weight=W.make_host_weight(rows, 16, seed=1))
    ht.start(lambda k: batches[k], len(batches))
    for k in range(len(batches)):
        o = ht.forward(k)
        ht.backward((o - 0.1).contiguous())
    ht.finish()
    print(name, "ok", ht.cache_stats())
    sys.exit(0)
mk, kw = CASES[name]
cfg = mk()
B = kw.get("batch", cfg.batch)
dev = torch.device("cuda", 0)
for fused in (True, False):
    emb = tt.TTEmbeddingBag.from_config(cfg, max_batch=B, fused_update=fused, fp32_cores=kw.get("fp32", False),
                                        optimizer="adagrad" if not fused else "sgd")
    emb.load_cores(W.make_cores(cfg, seed=1))
    idx, off = W.make_batch(cfg, seed=1, batch=B)
    out = emb.forward(torch.as_tensor(idx, device=dev), torch.as_tensor(off, device=dev), B)
    emb.backward(torch.as_tensor(W.make_grad_out(cfg, B, seed=1), device=dev), lr=0.01)
    if not fused:
        emb.update(0.01)
    torch.cuda.synchronize()
    assert emb.check() == 0
    print(name, "fused" if fused else "unfused", "ok", float(out.abs().sum()))
