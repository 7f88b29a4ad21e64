"""Multi-process host logic of the data-parallel path on CPU (gloo, world size 2).

Each rank takes its shard with `synth.workload.shard_batch`, computes its core gradients (the CPU
oracle stands in for the GPU kernels here: no GPU on this box), and the gradients are summed
with `parallel.allreduce_grads` (the same call bench.py uses with NCCL).  The result must
equal the full-batch gradients (R16: SUM, no 1/B), and SGD replicas must stay identical.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from synth import workload as W


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _cfg():
    return W.small_config([500, 90], [(8, 8, 8), (5, 5, 4)], (2, 2, 2), 4, 16, 3, 1.05)


def _worker(rank, world, port, result_path):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import Oracle
        from paper_conf_sc_wangwfmmd22_b200 import parallel
        cfg = _cfg()
        idx, off = W.make_batch(cfg, seed=2)
        cores = W.make_cores(cfg, seed=2)
        go = W.make_grad_out(cfg, cfg.batch, seed=2)
        li, lo, bl = W.shard_batch(idx, off, cfg.num_tables, cfg.batch, rank, world)
        orc = Oracle.from_config(cfg)
        g = orc.backward(cores, li, lo, bl, go[rank * bl:(rank + 1) * bl])
        flat = torch.cat([torch.from_numpy(x).reshape(-1) for tg in g for x in tg])
        parallel.allreduce_grads(flat)
        # every replica applies the same SGD step from the all-reduced gradients
        params = np.concatenate([x.reshape(-1) for c in cores for x in c]).astype(np.float32)
        new, _ = Oracle.update("sgd", 0.05, params, flat.numpy())
        gathered = [torch.zeros_like(torch.from_numpy(new)) for _ in range(world)]
        dist.all_gather(gathered, torch.from_numpy(new))
        if rank == 0:
            full = orc.backward(cores, idx, off, cfg.batch, go)
            ref = np.concatenate([x.reshape(-1) for tg in full for x in tg])
            ok_grad = np.allclose(flat.numpy(), ref, rtol=1e-12, atol=1e-12)
            ok_rep = all(torch.equal(gathered[0], x) for x in gathered)
            with open(result_path, "w") as f:
                f.write(f"{int(ok_grad)} {int(ok_rep)} {float(np.abs(flat.numpy() - ref).max())}")
    finally:
        dist.destroy_process_group()


def test_gloo_world2_allreduce_equals_full_batch(tmp_path):
    port = _free_port()
    res = tmp_path / "res.txt"
    mp.spawn(_worker, args=(2, port, str(res)), nprocs=2, join=True)
    ok_grad, ok_rep, err = res.read_text().split()
    assert ok_grad == "1", f"sharded SUM != full batch (max err {err})"
    assert ok_rep == "1"


def test_shard_bags_partition():
    from paper_conf_sc_wangwfmmd22_b200 import parallel
    cfg = _cfg()
    lens = np.random.default_rng(0).integers(0, 5, size=cfg.num_tables * cfg.batch)
    idx, off = W.make_batch(cfg, seed=1, lengths=lens)
    pieces = [W.shard_batch(idx, off, cfg.num_tables, cfg.batch, r, 4) for r in range(4)]
    assert sum(len(p[0]) for p in pieces) == len(idx)
    for r, (i, o, bl) in enumerate(pieces):
        assert bl == 4 and o[0] == 0 and o[-1] == len(i)
        for t in range(cfg.num_tables):           # bag (t, b) of the shard == bag (t, r*bl+b)
            for b in range(bl):
                gb = t * cfg.batch + r * bl + b
                np.testing.assert_array_equal(i[o[t * bl + b]:o[t * bl + b + 1]], idx[off[gb]:off[gb + 1]])
    with pytest.raises(ValueError):
        W.shard_batch(idx, off, cfg.num_tables, cfg.batch, 0, 3)


class _FakeEmb:
    """Host stand-in for TTEmbeddingBag in the GradSync host-logic test (no GPU here): flat
    padded cores / grads and an SGD update with the library's semantics (zero gradient = no
    change), via the oracle's update (fp64 -> fp32)."""

    def __init__(self, params, grads, n_pad):
        self.fused = False
        self.n_floats = len(params)
        self.cores = torch.zeros(n_pad)
        self.cores[:len(params)] = torch.from_numpy(params)
        self.grads = torch.zeros(n_pad)
        self.grads[:len(grads)] = torch.from_numpy(grads.astype(np.float32))
        self.device = torch.device("cpu")

    def grad_buckets(self):
        return [(0, 0), (0, self.n_floats), (0, 0)]

    def update(self, lr):
        self.update_range(lr, 0, self.n_floats)

    def update_range(self, lr, b, n):
        from oracle import Oracle
        e = min(b + n, self.n_floats)
        if e > b:
            p, _ = Oracle.update("sgd", lr, self.cores[b:e].numpy(), self.grads[b:e].double().numpy())
            self.cores[b:e] = torch.from_numpy(p)


def _sync_worker(rank, world, port, result_path, mode):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from oracle import Oracle
        from paper_conf_sc_wangwfmmd22_b200 import parallel
        cfg = _cfg()
        idx, off = W.make_batch(cfg, seed=3)
        cores = W.make_cores(cfg, seed=3)
        go = W.make_grad_out(cfg, cfg.batch, seed=3)
        li, lo, bl = W.shard_batch(idx, off, cfg.num_tables, cfg.batch, rank, world)
        orc = Oracle.from_config(cfg)
        g = orc.backward(cores, li, lo, bl, go[rank * bl:(rank + 1) * bl])
        flat_g = np.concatenate([x.reshape(-1) for tg in g for x in tg])
        params = np.concatenate([x.reshape(-1) for c in cores for x in c]).astype(np.float32)
        n_pad = -(-len(params) // 64) * 64
        emb = _FakeEmb(params, flat_g, n_pad)
        parallel.GradSync(emb, mode=mode).exchange_and_update(0.05)
        gathered = [torch.zeros(n_pad) for _ in range(world)]
        dist.all_gather(gathered, emb.cores)
        if rank == 0:
            full = orc.backward(cores, idx, off, cfg.batch, go)
            ref_g = np.concatenate([x.reshape(-1) for tg in full for x in tg])
            ref_p, _ = Oracle.update("sgd", 0.05, params, ref_g)
            got = gathered[0][:len(params)].numpy()
            ok = np.allclose(got, ref_p, rtol=1e-6, atol=1e-7)
            ok_rep = all(torch.equal(gathered[0], x) for x in gathered)
            ok_pad = float(gathered[0][len(params):].abs().sum()) == 0.0
            with open(result_path, "w") as f:
                f.write(f"{int(ok)} {int(ok_rep)} {int(ok_pad)} {float(np.abs(got - ref_p).max())}")
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["allreduce", "rs_ag"])
def test_gradsync_world2_equals_full_batch_update(tmp_path, mode):
    """parallel.GradSync: bucketed all-reduce + replicated update, and reduce-scatter
    + sharded update + all-gather, give every rank the full-batch SGD step (R16: SUM) and
    bitwise-identical replicas; the flat-buffer padding stays zero."""
    port = _free_port()
    res = tmp_path / "res.txt"
    mp.spawn(_sync_worker, args=(2, port, str(res), mode), nprocs=2, join=True)
    ok, ok_rep, ok_pad, err = res.read_text().split()
    assert ok == "1", f"{mode}: update != full-batch update (max err {err})"
    assert ok_rep == "1" and ok_pad == "1"


def test_shard_range():
    from paper_conf_sc_wangwfmmd22_b200 import parallel
    assert parallel.shard_range(1024, 4, 3) == (768, 256)
    with pytest.raises(ValueError):
        parallel.shard_range(1000, 3, 0)
