"""Host-memory tier (PAPER §V), CPU part.

* The oracle (oracle/hosttier_ref.py) pinned to torch.nn.EmbeddingBag + autograd + SGD (float64)
  and to the pipeline invariants (queue length 1 is sequential; without the cache a pipeline
  differs from sequential training exactly when consecutive batches share rows).
* The parameter server's native host code (ttemb_ht_host_gather / ttemb_ht_host_sgd) bit-exact
  against the oracle's SGD, and its index preparation (prepare_batch) against its definition.
"""
import ctypes as C

import numpy as np
import pytest
import torch

from oracle import hosttier_ref as HR
from synth import workload as W

ROWS = [300, 50, 800]
DIM = 8
B = 16
POOL = 3
TB = np.concatenate([[0], np.cumsum(ROWS)]).astype(np.int64)


def _batches(n, s=1.05, seed=0):
    return [W.make_host_batch(ROWS, B, POOL, s, step=k, seed=seed) for k in range(n)]


def _gos(n, seed=0):
    return [W.make_host_grad_out(len(ROWS), B, DIM, step=k, seed=seed) for k in range(n)]


def _targets(n, seed=0):
    return HR.squared_loss_grad([0.1 * g for g in _gos(n, seed)])


def test_oracle_matches_torch_embeddingbag_training():
    """3 SGD steps of the oracle == nn.EmbeddingBag(sum) + autograd + optim.SGD in float64."""
    W0 = W.make_host_weight(ROWS, DIM, seed=1)
    bs, gs = _batches(3), _gos(3)
    lr = 0.1
    Wq, outs = HR.train_sequential(W0, TB, bs, HR.squared_loss_grad(gs), B, lr)
    emb = torch.nn.EmbeddingBag(int(TB[-1]), DIM, mode="sum").double()
    with torch.no_grad():
        emb.weight.copy_(torch.from_numpy(W0.astype(np.float64)))
    opt = torch.optim.SGD(emb.parameters(), lr=lr)
    T = len(ROWS)
    for (idx, off), go, out in zip(bs, gs, outs):
        bag = np.repeat(np.arange(T * B), np.diff(off))
        gidx = idx + TB[:-1][bag // B]
        o = emb(torch.from_numpy(gidx), torch.from_numpy(off[:-1]))          # [T*B][N], bag t*B+b
        ref = o.view(T, B, DIM).permute(1, 0, 2)
        np.testing.assert_allclose(out, ref.detach().numpy(), rtol=1e-5, atol=1e-6)
        opt.zero_grad()
        (0.5 * (ref - torch.from_numpy(go.astype(np.float64))) ** 2).sum().backward()
        opt.step()
    np.testing.assert_allclose(Wq, emb.weight.detach().numpy(), rtol=1e-5, atol=1e-6)


def test_oracle_row_grads_and_step_single_occurrence():
    """One position per bag, distinct rows: g_r = grad_out[b][t] and W_r <- W_r - lr g_r."""
    W0 = W.make_host_weight(ROWS, DIM, seed=2)
    T = len(ROWS)
    idx = np.concatenate([np.arange(B) * 7 % ROWS[t] for t in range(T)]).astype(np.int64)
    off = np.arange(T * B + 1, dtype=np.int64)
    go = _gos(1, seed=3)[0]
    rows, g = HR.row_grads(go, TB, idx, off, B)
    assert len(rows) == T * B
    for t in range(T):
        for b in range(B):
            r = TB[t] + idx[t * B + b]
            np.testing.assert_array_equal(g[np.searchsorted(rows, r)], go[b, t])
    out = HR.forward(W0, TB, idx, off, B)
    for t in range(T):
        np.testing.assert_array_equal(out[:, t], W0[TB[t] + idx[t * B:(t + 1) * B]])


def test_stale_pipeline_invariants():
    W0 = W.make_host_weight(ROWS, DIM, seed=4)
    bs, gs = _batches(6), _targets(6)
    seq, so = HR.train_sequential(W0, TB, bs, gs, B, 0.05)
    s1, o1 = HR.train_stale(W0, TB, bs, gs, B, 0.05, L=1)
    np.testing.assert_array_equal(s1, seq)                     # L = 1 is sequential
    for a, b in zip(o1, so):
        np.testing.assert_array_equal(a, b)
    s3, o3 = HR.train_stale(W0, TB, bs, gs, B, 0.05, L=3)      # Zipf: hot rows repeat
    assert not np.array_equal(s3, seq)
    assert not np.array_equal(o3[1], so[1])                    # batch 1 read rows batch 0 updated
    np.testing.assert_array_equal(o3[0], so[0])                # batch 0 cannot be stale
    # batches touching disjoint rows: no RAW hazard, stale == sequential for any L
    T = len(ROWS)
    dis = []
    for k in range(4):       # batch k uses rows [48k, 48k+48) of every table (all tables >= 50 rows
        idx = np.concatenate([(np.arange(B * POOL) + k * B * POOL) % ROWS[t] for t in range(T)])
        dis.append((idx.astype(np.int64), np.arange(T * B + 1, dtype=np.int64) * POOL))
    g4 = _targets(4, seed=5)
    for L in (2, 3):
        a, oa = HR.train_stale(W0, TB, dis, g4, B, 0.05, L=L)
        b, ob = HR.train_sequential(W0, TB, dis, g4, B, 0.05)
        shared = [any(np.intersect1d(dis[k][0][t * B * POOL:(t + 1) * B * POOL],
                                     dis[j][0][t * B * POOL:(t + 1) * B * POOL]).size for t in range(T))
                  for k in range(4) for j in range(k + 1, min(4, k + L))]
        if not any(shared):
            np.testing.assert_array_equal(a, b)
        for k in range(4):
            hazard = any(np.intersect1d(dis[k][0][t * B * POOL:(t + 1) * B * POOL],
                                        dis[j][0][t * B * POOL:(t + 1) * B * POOL]).size
                         for t in range(T) for j in range(max(0, k - L + 1), k))
            if not hazard:
                np.testing.assert_array_equal(oa[k], ob[k])


def test_host_gather_and_sgd_native_bit_exact():
    import paper_conf_sc_wangwfmmd22_b200  # noqa: F401  (loads libttemb.so)
    from paper_conf_sc_wangwfmmd22_b200 import _lib as L
    lib = L.load()
    n_rows = int(TB[-1])
    Wt = W.make_host_weight(ROWS, DIM, seed=6)
    ids = np.array(sorted(np.random.default_rng(0).choice(n_rows, 97, replace=False)), dtype=np.int64)
    out = np.empty((len(ids), DIM), dtype=np.float32)
    for nth in (1, 3, 0):
        assert lib.ttemb_ht_host_gather(Wt.ctypes.data, n_rows, DIM, ids.ctypes.data, len(ids),
                                        out.ctypes.data, nth) == 0
        np.testing.assert_array_equal(out, Wt[ids])
    g = np.random.default_rng(1).uniform(-3, 3, size=(len(ids), DIM)).astype(np.float32)
    for nth in (1, 4):
        a = Wt.copy()
        assert lib.ttemb_ht_host_sgd(a.ctypes.data, n_rows, DIM, ids.ctypes.data, len(ids), g.ctypes.data,
                                     C.c_float(0.37), nth) == 0
        ref = Wt.copy()
        HR.sgd(ref, ids, g, 0.37)
        np.testing.assert_array_equal(a, ref)
    bad = np.array([0, n_rows], dtype=np.int64)
    a = Wt.copy()
    assert lib.ttemb_ht_host_gather(Wt.ctypes.data, n_rows, DIM, bad.ctypes.data, 2, out.ctypes.data, 1) == -3
    assert lib.ttemb_ht_host_sgd(a.ctypes.data, n_rows, DIM, bad.ctypes.data, 2, g.ctypes.data,
                                 C.c_float(1.0), 1) == -3
    np.testing.assert_array_equal(a, Wt)                        # nothing written
    assert lib.ttemb_ht_host_gather(None, n_rows, DIM, ids.ctypes.data, 1, out.ctypes.data, 1) == -1


def test_prepare_batch_definition():
    from paper_conf_sc_wangwfmmd22_b200.hosttier import prepare_batch
    idx, off = _batches(1)[0]
    hb = prepare_batch(idx, off, TB, B)
    T = len(ROWS)
    bag = np.repeat(np.arange(T * B), np.diff(off))
    gid = idx + TB[:-1][bag // B]
    np.testing.assert_array_equal(hb.ids, np.unique(gid))
    np.testing.assert_array_equal(hb.ids[hb.ridx], gid)                # block row of each position
    for u in range(len(hb.ids)):
        pos = np.nonzero(gid == hb.ids[u])[0]                            # position order
        np.testing.assert_array_equal(hb.occ_bag[hb.occ_ptr[u]:hb.occ_ptr[u + 1]], bag[pos])
    with pytest.raises(ValueError):
        prepare_batch(np.full_like(idx, ROWS[0]), off, TB, B)           # id outside table 0
