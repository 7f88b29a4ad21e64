"""Data-parallel path through the CUDA kernels, two ranks sharing one GPU over gloo
(the box has one B200; NCCL needs one GPU per rank).  Every rank runs the C ABI forward /
unfused backward on its shard of the global batch, `parallel.GradSync` exchanges the gradients
(bucketed all-reduce, or reduce-scatter -> sharded update -> all-gather), and after three SGD
steps the replicas must be bitwise identical and equal the oracle's full-batch trajectory."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from synth import workload as W

pytestmark = pytest.mark.gpu

CASES = {
    "tc-r64": lambda: W.small_config([20000, 300], [(28, 28, 26), (7, 7, 7)], (4, 4, 4), 64, 96, 1, 1.05),
    "ffma-r8": lambda: W.small_config([1000, 200], [(10, 10, 10), (6, 6, 6)], (2, 2, 4), 8, 64, 2, 1.05),
}


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, res, case, mode):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_sc_wangwfmmd22_b200 as tt
        from paper_conf_sc_wangwfmmd22_b200 import parallel
        from oracle import Oracle
        torch.cuda.set_device(0)
        dev = torch.device("cuda", 0)
        cfg = CASES[case]()
        B = cfg.batch
        bl = B // world
        cores = W.make_cores(cfg, seed=8)
        emb = tt.TTEmbeddingBag.from_config(cfg, max_batch=bl, max_nnz=bl * cfg.num_tables * cfg.pooling,
                                            fused_update=False)
        emb.load_cores(cores)
        sync = parallel.GradSync(emb, mode=mode)
        lr = 0.05
        for s in range(3):
            idx, off = W.make_batch(cfg, step=s, seed=8)
            go = W.make_grad_out(cfg, B, step=s, seed=8)
            li, lo, _ = W.shard_batch(idx, off, cfg.num_tables, B, rank, world)
            emb.forward(torch.as_tensor(li, device=dev), torch.as_tensor(lo, device=dev), bl)
            emb.backward(torch.as_tensor(go[rank * bl:(rank + 1) * bl].copy(), device=dev))
            sync.exchange_and_update(lr)
        torch.cuda.synchronize()
        assert emb.check() == 0
        mine = emb.cores.cpu()
        parts = [torch.empty_like(mine) for _ in range(world)]
        dist.all_gather(parts, mine)
        if rank == 0:
            orc = Oracle.from_config(cfg)
            ref = [tuple(x.copy() for x in c) for c in cores]
            for s in range(3):
                idx, off = W.make_batch(cfg, step=s, seed=8)
                go = W.make_grad_out(cfg, B, step=s, seed=8)
                g = orc.backward(ref, idx, off, B, go)
                ref = [tuple(Oracle.update("sgd", lr, c[k], g[t][k])[0] for k in range(3)) for t, c in enumerate(ref)]
            ok_rep = all(torch.equal(parts[0], p) for p in parts)
            errs = []
            for t, cv in enumerate(emb.core_views()):
                for k in range(3):
                    got = cv[k].cpu().numpy()
                    if not np.allclose(got, ref[t][k], rtol=1e-4, atol=1e-5):
                        errs.append(f"t{t} C{k + 1} max err {np.abs(got - ref[t][k]).max():.3g}")
            with open(res, "w") as f:
                f.write(f"{int(ok_rep)}|{';'.join(errs)}")
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["allreduce", "rs_ag"])
@pytest.mark.parametrize("case", list(CASES))
def test_two_ranks_one_gpu_trajectory(tmp_path, case, mode):
    res = tmp_path / "res.txt"
    mp.spawn(_worker, args=(2, _free_port(), str(res), case, mode), nprocs=2, join=True)
    ok_rep, errs = res.read_text().split("|")
    assert ok_rep == "1", "replicas differ"
    assert errs == "", errs
