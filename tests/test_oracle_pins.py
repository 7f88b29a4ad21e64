"""Pins for the CPU oracle (oracle/), against things other than itself.

Every pin cites the passage it checks.  None of these tests touches the CUDA
path.  A plausible mistake in the oracle (swapped digit order, transposed
core operand, dropped term, wrong bag/table mapping, wrong update sign) fails
at least one of them:

  * Fig. 5(b) worked example                     -> digit order, prefix sharing
  * R = 1 closed form (np.kron)                          -> column order, slice choice
  * TT-SVD round trip (np.linalg.svd, full TT ranks)     -> Eq. 2 / Eq. 3 end to end
  * identity cores -> plain table, torch embedding_bag   -> Eq. 4 pooling, offsets, empty bags
  * numpy unique / stable argsort / unravel_index        -> integer plan
  * exact central differences on integer data            -> gradients (L linear per core)
  * torch.autograd through a dense materialisation       -> gradients
  * torch.optim.SGD / Adagrad                            -> update rule
"""
import json
import os

import numpy as np
import pytest
import torch

from oracle import Oracle, OracleError, ERR_INDEX_RANGE, ERR_INVALID
from synth import workload as W

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def tiny_cfg(rows=(1000,), factors=((10, 10, 10),), col=(2, 2, 4), R=8, B=64, L=1, s=None):
    return W.small_config(rows, factors, col, R, B, L, s)


def materialise_torch(cores_t, row_factors, col, M):
    """Dense W[M][N] from TT cores via torch.einsum (fp64); digits through
    np.unravel_index (big-endian mixed radix)."""
    c1, c2, c3 = cores_t
    m1, m2, m3 = row_factors
    i1, i2, i3 = np.unravel_index(np.arange(M), (m1, m2, m3))
    a = c1[torch.as_tensor(i1)]          # [M][n1][R]
    b = c2[torch.as_tensor(i2)]          # [M][R][n2][R]
    c = c3[torch.as_tensor(i3)]          # [M][R][n3]
    w = torch.einsum("mjr,mrks,msl->mjkl", a, b, c)
    return w.reshape(M, -1)


# ---------------------------------------------------------------------------
# Digits and the worked example
# ---------------------------------------------------------------------------
def test_fig5b_worked_example():
    g = json.load(open(os.path.join(GOLD, "fig5b.json")))
    m = tuple(g["row_factors"])
    orc = Oracle([8], [m], (1, 1, 2), 2)
    for i, want in zip(g["ids"], g["tt_indices"]):
        assert orc.digits(0, i) == tuple(want)
    # one bag holding both ids: 2 unique rows, 1 shared prefix (Reuse buffer)
    plan = orc.plan(np.array(g["ids"]), np.array([0, 2]), 1)
    assert plan["U"] == 2 and plan["P"] == g["unique_prefixes"]


def test_digits_match_unravel_index():
    orc = Oracle([1000, 7 * 5 * 3], [(10, 10, 10), (7, 5, 3)], (1, 1, 1), 1)
    for t, m in enumerate([(10, 10, 10), (7, 5, 3)]):
        for i in range(0, int(np.prod(m)), 7):
            assert orc.digits(t, i) == tuple(int(x) for x in np.unravel_index(i, m))


# ---------------------------------------------------------------------------
# Forward
# ---------------------------------------------------------------------------
def test_rank1_kronecker_closed_form():
    cfg = W.small_config([60], [(3, 4, 5)], (2, 3, 2), 1, 1)
    cores = W.make_cores(cfg, seed=3)
    c1, c2, c3 = cores[0]
    orc = Oracle.from_config(cfg)
    for i in range(60):
        i1, i2, i3 = np.unravel_index(i, (3, 4, 5))
        want = np.kron(np.kron(c1[i1, :, 0].astype(np.float64), c2[i2, 0, :, 0]), c3[i3, 0, :])
        for literal in (False, True):
            np.testing.assert_allclose(orc.row(cores, 0, i, literal), want, rtol=1e-14, atol=0)


def test_tt_svd_round_trip():
    """Dense W (M=8 x N=8) -> TT-SVD with full ranks (R=4) -> oracle rows == W."""
    m, n, R = (2, 2, 2), (2, 2, 2), 4
    rng = np.random.default_rng(0)
    Wd = rng.standard_normal((8, 8))
    X = Wd.reshape(*m, *n).transpose(0, 3, 1, 4, 2, 5)        # (i1 j1)(i2 j2)(i3 j3)
    U1, S1, V1 = np.linalg.svd(X.reshape(m[0] * n[0], -1), full_matrices=False)
    assert U1.shape[1] == R
    rest = (S1[:, None] * V1).reshape(R * m[1] * n[1], m[2] * n[2])
    U2, S2, V2 = np.linalg.svd(rest, full_matrices=False)
    assert U2.shape[1] == R
    c1 = U1.reshape(m[0], n[0], R)
    c2 = U2.reshape(R, m[1], n[1], R).transpose(1, 0, 2, 3)
    c3 = (S2[:, None] * V2).reshape(R, m[2], n[2]).transpose(1, 0, 2)
    cores = [(c1.astype(np.float32), c2.astype(np.float32), c3.astype(np.float32))]
    orc = Oracle([8], [m], n, R)
    out = orc.forward(cores, np.arange(8), np.arange(9), 8)      # one row per bag
    np.testing.assert_allclose(out[:, 0, :], Wd, atol=2e-6 * np.abs(Wd).max())
    for literal in (True,):
        out_l = orc.forward(cores, np.arange(8), np.arange(9), 8, literal=literal)
        np.testing.assert_allclose(out_l, out, rtol=1e-12, atol=1e-14)


def test_identity_cores_is_plain_embedding_bag():
    """m=(M,1,1), n=(N,1,1), C2[0]=I, C3[0]=e_1  ->  W = C1[:, :, 0] (a plain table)."""
    M, N, R, B = 50, 6, 3, 12
    rng = np.random.default_rng(1)
    c1 = rng.standard_normal((M, N, R)).astype(np.float32)
    c2 = np.eye(R, dtype=np.float32).reshape(1, R, 1, R)
    c3 = np.zeros((1, R, 1), np.float32); c3[0, 0, 0] = 1.0
    lens = rng.integers(0, 5, size=B); lens[3] = 0; lens[-1] = 0   # empty bags
    off = np.concatenate([[0], np.cumsum(lens)]).astype(np.int64)
    idx = rng.integers(0, M, size=int(off[-1])).astype(np.int64)
    idx[:3] = idx[0]                                               # duplicates in a bag
    orc = Oracle([M], [(M, 1, 1)], (N, 1, 1), R)
    out = orc.forward([(c1, c2, c3)], idx, off, B)
    ref = torch.nn.functional.embedding_bag(torch.as_tensor(idx), torch.as_tensor(c1[:, :, 0], dtype=torch.float64),
                                            torch.as_tensor(off[:-1]), mode="sum")
    np.testing.assert_array_equal(out[:, 0, :], ref.numpy())


def test_forward_matches_dense_embedding_bag_multitable():
    cfg = W.small_config([37, 100, 5], [(3, 4, 4), (5, 4, 5), (1, 2, 3)], (2, 3, 2), 5, 9, 1, 1.05)
    rng = np.random.default_rng(2)
    T, B = cfg.num_tables, cfg.batch
    lens = rng.integers(0, 6, size=T * B); lens[0] = 0
    idx, off = W.make_batch(cfg, step=1, seed=5, lengths=lens)
    cores = W.make_cores(cfg, seed=5)
    orc = Oracle.from_config(cfg)
    out = orc.forward(cores, idx, off, B)
    for t in range(T):
        Wt = materialise_torch([torch.as_tensor(x, dtype=torch.float64) for x in cores[t]],
                               cfg.row_factors[t], cfg.col_factors, cfg.table_rows[t])
        o = off[t * B:(t + 1) * B + 1]
        ref = torch.nn.functional.embedding_bag(torch.as_tensor(idx[o[0]:o[-1]]), Wt,
                                                torch.as_tensor(o[:-1] - o[0]), mode="sum")
        np.testing.assert_allclose(out[:, t, :], ref.numpy(), rtol=1e-12, atol=1e-13)


def test_forward_literal_equals_chain():
    cfg = tiny_cfg()
    idx, off = W.make_batch(cfg, seed=1)
    cores = W.make_cores(cfg, seed=1)
    orc = Oracle.from_config(cfg)
    a = orc.forward(cores, idx, off, cfg.batch)
    b = orc.forward(cores, idx, off, cfg.batch, literal=True)
    np.testing.assert_allclose(a, b, rtol=1e-12, atol=1e-14)


def test_index_range_and_offsets_errors():
    orc = Oracle([10], [(2, 2, 3)], (1, 1, 2), 2)
    cores = [(np.ones((2, 1, 2), np.float32), np.ones((2, 2, 1, 2), np.float32), np.ones((3, 2, 2), np.float32))]
    with pytest.raises(OracleError) as e:          # 10 <= id < 12 is padding, invalid (R10)
        orc.forward(cores, np.array([10]), np.array([0, 1]), 1)
    assert e.value.code == ERR_INDEX_RANGE
    with pytest.raises(OracleError) as e:
        orc.forward(cores, np.array([-1]), np.array([0, 1]), 1)
    assert e.value.code == ERR_INDEX_RANGE
    with pytest.raises(OracleError) as e:          # offsets[-1] != nnz
        orc.forward(cores, np.array([1, 2]), np.array([0, 1]), 1)
    assert e.value.code == ERR_INVALID


# ---------------------------------------------------------------------------
# Plan
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("name,seed", [("c1", 1), ("c2", 2)])
def test_plan_matches_numpy(name, seed):
    cfg = W.config(name)
    B = min(cfg.batch, 512)
    idx, off = W.make_batch(cfg, seed=seed, batch=B)
    orc = Oracle.from_config(cfg)
    plan = orc.plan(idx, off, B)
    T = cfg.num_tables
    # group-major plan key (R29): digits by numpy, re-ravelled in (i2, i1, i3) order
    mf = np.array(cfg.row_factors, np.int64)
    span = mf.prod(axis=1)
    gbase = np.concatenate([[0], np.cumsum(span)[:-1]]).astype(np.int64)
    bag = np.repeat(np.arange(T * B), np.diff(off))
    tab = bag // B
    d1, d2, d3 = (np.array(x, np.int64) for x in zip(*[np.unravel_index(i, tuple(mf[t])) for i, t in zip(idx, tab)]))
    key = gbase[tab] + (d2 * mf[tab, 0] + d1) * mf[tab, 2] + d3
    order = np.argsort(key, kind="stable")
    np.testing.assert_array_equal(plan["skey"], key[order])
    np.testing.assert_array_equal(plan["spos"], order)
    np.testing.assert_array_equal(plan["bag_of"], (bag % B) * T + tab)
    uk, inv, cnt = np.unique(key, return_inverse=True, return_counts=True)
    np.testing.assert_array_equal(plan["ukey"], uk)
    np.testing.assert_array_equal(plan["inverse"], inv)
    np.testing.assert_array_equal(plan["seg_off"], np.concatenate([[0], np.cumsum(cnt)]))
    # every unique row's digits (from the first position that holds it)
    firstpos = order[np.concatenate([[0], np.cumsum(cnt)[:-1]])]
    ut, i1, i2, i3 = tab[firstpos], d1[firstpos], d2[firstpos], d3[firstpos]
    np.testing.assert_array_equal(plan["row_i3"], i3)
    pk = np.stack([ut, i2, i1], 1)
    upk, pinv = np.unique(pk, axis=0, return_inverse=True)
    np.testing.assert_array_equal(plan["row_pfx"], pinv.ravel())
    assert plan["P"] == len(upk)
    first = np.concatenate([[0], np.flatnonzero(np.diff(pinv.ravel())) + 1])
    np.testing.assert_array_equal(plan["pfx_t"], upk[:, 0])
    np.testing.assert_array_equal(plan["pfx_i2"], upk[:, 1])
    np.testing.assert_array_equal(plan["pfx_i1"], upk[:, 2])
    np.testing.assert_array_equal(plan["row_seg"], np.concatenate([first, [len(uk)]]))
    np.testing.assert_array_equal(plan["grp_pfx"], np.arange(plan["P"]))
    gu, gfirst = np.unique(upk[:, :2], axis=0, return_index=True)
    assert plan["NG"] == len(gu)
    np.testing.assert_array_equal(plan["grp_off"], np.concatenate([gfirst, [plan["P"]]]))
    np.testing.assert_array_equal(plan["grp_t"], gu[:, 0])
    np.testing.assert_array_equal(plan["grp_i2"], gu[:, 1])


@pytest.mark.parametrize("name,seed", [("c2", 3), ("c3", 4)])
def test_plan_key_is_a_bijection_of_table_row(name, seed):
    """DESIGN.md R29: the plan's distinct keys, mapped back to (table, row) by inverting the key
    K = kbase_t + (i2 m1 + i1) m3 + i3 and re-composing row = (i1 m2 + i2) m3 + i3 (Eq. 3), are
    exactly the distinct (t, row) pairs of the batch: np.unique(rowbase_t + id) (SURVEY 8(c)'s
    plan definition), and ukey is ascending in (t, i2, i1, i3) order."""
    cfg = W.config(name)
    B = min(cfg.batch, 1024)
    idx, off = W.make_batch(cfg, seed=seed, batch=B)
    plan = Oracle.from_config(cfg).plan(idx, off, B)
    T = cfg.num_tables
    mf = np.array(cfg.row_factors, np.int64)
    rows = np.array(cfg.table_rows, np.int64)
    kbase = np.concatenate([[0], np.cumsum(mf.prod(axis=1))])
    rowbase = np.concatenate([[0], np.cumsum(rows)])
    uk = plan["ukey"].astype(np.int64)
    t = np.searchsorted(kbase, uk, side="right") - 1
    local = uk - kbase[t]
    i3 = local % mf[t, 2]
    i1 = (local // mf[t, 2]) % mf[t, 0]
    i2 = (local // mf[t, 2]) // mf[t, 0]
    row = (i1 * mf[t, 1] + i2) * mf[t, 2] + i3
    assert (row < rows[t]).all()
    tab = np.repeat(np.arange(T * B), np.diff(off)) // B
    want = np.unique(rowbase[tab] + np.asarray(idx, np.int64))
    np.testing.assert_array_equal(np.sort(rowbase[t] + row), want)
    order = np.lexsort((i3, i1, i2, t))
    np.testing.assert_array_equal(order, np.arange(len(uk)))


def test_plan_empty_batch():
    orc = Oracle([10, 20], [(2, 2, 3), (3, 3, 3)], (1, 1, 2), 2)
    plan = orc.plan(np.zeros(0, np.int64), np.zeros(2 * 4 + 1, np.int64), 4)
    assert plan["U"] == 0 and plan["P"] == 0 and plan["NG"] == 0
    assert list(plan["seg_off"]) == [0] and list(plan["row_seg"]) == [0]


# ---------------------------------------------------------------------------
# Backward
# ---------------------------------------------------------------------------
def _int_case(seed):
    cfg = W.small_config([30, 12], [(3, 2, 5), (2, 3, 2)], (2, 1, 3), 3, 7, 1)
    rng = np.random.default_rng(seed)
    cores = [tuple(rng.integers(-2, 3, size=np.shape(x)).astype(np.float32) for x in c)
             for c in W.make_cores(cfg)]
    lens = rng.integers(0, 4, size=cfg.num_tables * cfg.batch)
    idx, off = W.make_batch(cfg, seed=seed, lengths=lens)
    go = rng.integers(-2, 3, size=(cfg.batch, cfg.num_tables, cfg.dim)).astype(np.float32)
    return cfg, cores, idx, off, go


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_gradients_exact_central_differences(seed):
    """L is linear in each core, so (L(C+D) - L(C-D)) / 2 = <dL/dC, D> exactly;
    integer data keeps every fp64 operation exact."""
    cfg, cores, idx, off, go = _int_case(seed)
    orc = Oracle.from_config(cfg)
    B = cfg.batch
    grads = orc.backward(cores, idx, off, B, go)
    grads_l = orc.backward(cores, idx, off, B, go, literal=True)
    rng = np.random.default_rng(100 + seed)

    def loss(cs):
        return float((orc.forward(cs, idx, off, B) * go.astype(np.float64)).sum())

    for t in range(cfg.num_tables):
        for k in range(3):
            D = rng.integers(-1, 2, size=cores[t][k].shape).astype(np.float32)
            cp = [list(c) for c in cores]
            cm = [list(c) for c in cores]
            cp[t][k] = cores[t][k] + D
            cm[t][k] = cores[t][k] - D
            fd = (loss(cp) - loss(cm)) / 2.0
            assert fd == float((grads[t][k] * D).sum())
            np.testing.assert_array_equal(grads[t][k], grads_l[t][k])


@pytest.mark.parametrize("L,s", [(1, 1.05), (4, None)])
def test_gradients_match_autograd(L, s):
    cfg = W.small_config([200, 64], [(5, 6, 7), (4, 4, 4)], (2, 2, 3), 4, 16, L, s)
    idx, off = W.make_batch(cfg, seed=3)
    cores = W.make_cores(cfg, seed=3)
    go = W.make_grad_out(cfg, cfg.batch, seed=3)
    orc = Oracle.from_config(cfg)
    grads = orc.backward(cores, idx, off, cfg.batch, go)
    B = cfg.batch
    for t in range(cfg.num_tables):
        ct = [torch.tensor(x, dtype=torch.float64, requires_grad=True) for x in cores[t]]
        Wt = materialise_torch(ct, cfg.row_factors[t], cfg.col_factors, cfg.table_rows[t])
        o = off[t * B:(t + 1) * B + 1]
        out = torch.nn.functional.embedding_bag(torch.as_tensor(idx[o[0]:o[-1]]), Wt,
                                                torch.as_tensor(o[:-1] - o[0]), mode="sum")
        (out * torch.as_tensor(go[:, t, :], dtype=torch.float64)).sum().backward()
        for k in range(3):
            np.testing.assert_allclose(grads[t][k], ct[k].grad.numpy(), rtol=1e-11, atol=1e-12)


def test_gradients_shard_sum_invariant():
    """Sum of per-shard gradients == full-batch gradients (SUM allreduce, R16)."""
    cfg = W.small_config([500], [(8, 8, 8)], (2, 2, 2), 4, 32, 3, 1.05)
    idx, off = W.make_batch(cfg, seed=4)
    cores = W.make_cores(cfg, seed=4)
    go = W.make_grad_out(cfg, cfg.batch, seed=4)
    orc = Oracle.from_config(cfg)
    full = orc.backward(cores, idx, off, cfg.batch, go)
    G = 4
    acc = None
    for r in range(G):
        i, o, bl = W.shard_batch(idx, off, 1, cfg.batch, r, G)
        g = orc.backward(cores, i, o, bl, go[r * bl:(r + 1) * bl])
        acc = g if acc is None else [tuple(a + b for a, b in zip(x, y)) for x, y in zip(acc, g)]
    for k in range(3):
        np.testing.assert_allclose(acc[0][k], full[0][k], rtol=1e-12, atol=1e-12)


# ---------------------------------------------------------------------------
# Update
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("opt", ["sgd", "adagrad"])
def test_update_matches_torch_optim(opt):
    rng = np.random.default_rng(7)
    p0 = rng.standard_normal(1000).astype(np.float32)
    g1 = rng.standard_normal(1000); g1[::10] = 0.0
    g2 = rng.standard_normal(1000)
    lr, eps = 0.01, 1e-10
    pt = torch.tensor(p0, dtype=torch.float64, requires_grad=True)
    o = (torch.optim.SGD([pt], lr=lr) if opt == "sgd"
         else torch.optim.Adagrad([pt], lr=lr, eps=eps, initial_accumulator_value=0.0))
    p, s = p0, None
    for g in (g1, g2):
        pt.grad = torch.tensor(g)
        o.step()
        p, s = Oracle.update(opt, lr, p, g, s, eps)
        # the oracle rounds to fp32 once per step; feed torch the same rounded value
        with torch.no_grad():
            pt.copy_(torch.tensor(p, dtype=torch.float64))
        if opt == "adagrad":
            st = o.state[pt]["sum"].numpy()
            np.testing.assert_allclose(s, st, rtol=1e-7)
            o.state[pt]["sum"].copy_(torch.tensor(s, dtype=torch.float64))
    # re-run one step and compare values before rounding
    pt2 = torch.tensor(p0, dtype=torch.float64, requires_grad=True)
    o2 = (torch.optim.SGD([pt2], lr=lr) if opt == "sgd"
          else torch.optim.Adagrad([pt2], lr=lr, eps=eps, initial_accumulator_value=0.0))
    pt2.grad = torch.tensor(g1)
    o2.step()
    p1, _ = Oracle.update(opt, lr, p0, g1, None, eps)
    np.testing.assert_array_equal(p1, pt2.detach().numpy().astype(np.float32))
    assert np.array_equal(p1[::10], p0[::10])      # zero gradient leaves the slice unchanged


# ---------------------------------------------------------------------------
# Runtime index bijection (Sec. IV-B)
# ---------------------------------------------------------------------------
def test_bijection_is_a_row_permutation_of_the_dense_table():
    """New_Batch = {index(i_j)}: looking up i through the bijection reads row index(i) of
    the TT table, i.e. the bag sums of the dense table with rows permuted, W'[i] = W[index(i)]
    (numpy fancy indexing + torch embedding_bag; an inverse-map or per-table mix-up fails)."""
    cfg = W.small_config([37, 100, 5], [(3, 4, 4), (5, 4, 5), (1, 2, 3)], (2, 3, 2), 5, 9, 2, 1.05)
    rng = np.random.default_rng(7)
    T, B = cfg.num_tables, cfg.batch
    idx, off = W.make_batch(cfg, step=2, seed=7)
    cores = W.make_cores(cfg, seed=7)
    bij = [rng.permutation(M) for M in cfg.table_rows]
    orc = Oracle.from_config(cfg)
    out = orc.forward(cores, orc.apply_bijection(bij, idx, off, B), off, B)
    for t in range(T):
        Wt = materialise_torch([torch.as_tensor(x, dtype=torch.float64) for x in cores[t]],
                               cfg.row_factors[t], cfg.col_factors, cfg.table_rows[t])
        Wp = Wt[torch.as_tensor(bij[t])]
        o = off[t * B:(t + 1) * B + 1]
        ref = torch.nn.functional.embedding_bag(torch.as_tensor(idx[o[0]:o[-1]]), Wp,
                                                torch.as_tensor(o[:-1] - o[0]), mode="sum")
        np.testing.assert_allclose(out[:, t, :], ref.numpy(), rtol=1e-12, atol=1e-13)


def test_bijection_range_errors():
    orc = Oracle([10], [(2, 2, 3)], (1, 1, 2), 2)
    with pytest.raises(OracleError) as e:          # mapped id outside [0, M)
        orc.apply_bijection([np.array([0, 1, 2, 3, 4, 5, 6, 7, 8, 10])], np.array([9]), np.array([0, 1]), 1)
    assert e.value.code == ERR_INDEX_RANGE
    with pytest.raises(OracleError) as e:          # raw id outside [0, M)
        orc.apply_bijection([np.arange(10)], np.array([10]), np.array([0, 1]), 1)
    assert e.value.code == ERR_INDEX_RANGE
    np.testing.assert_array_equal(orc.apply_bijection([np.arange(10)[::-1]], np.array([0, 9, 3]),
                                                      np.array([0, 3]), 1), [9, 0, 6])


# ---------------------------------------------------------------------------
# nn.EmbeddingBag pooling variants (drop-in replacement, P:48 / P:306): mean, per-sample weights
# ---------------------------------------------------------------------------
@pytest.mark.parametrize("mode,weighted", [("mean", False), ("sum", True)])
def test_mean_and_weighted_bags_match_torch_embedding_bag(mode, weighted):
    """Forward and core gradients of mean / per-sample-weighted bags against
    torch.nn.functional.embedding_bag(mode, per_sample_weights) on the dense materialised table,
    differentiated by torch.autograd (variable bag lengths incl. empty bags)."""
    cfg = W.small_config([200, 64], [(5, 6, 7), (4, 4, 4)], (2, 2, 3), 4, 16, 1, 1.05)
    rng = np.random.default_rng(11)
    T, B = cfg.num_tables, cfg.batch
    lens = rng.integers(0, 6, size=T * B); lens[0] = 0; lens[5] = 0
    idx, off = W.make_batch(cfg, step=1, seed=11, lengths=lens)
    psw = rng.uniform(-2, 2, size=len(idx)).astype(np.float32) if weighted else None
    cores = W.make_cores(cfg, seed=11)
    go = W.make_grad_out(cfg, B, seed=11)
    orc = Oracle.from_config(cfg)
    out = orc.forward(cores, idx, off, B, per_sample_weights=psw, mode=mode)
    grads = orc.backward(cores, idx, off, B, go, per_sample_weights=psw, mode=mode)
    for t in range(T):
        ct = [torch.tensor(x, dtype=torch.float64, requires_grad=True) for x in cores[t]]
        Wt = materialise_torch(ct, cfg.row_factors[t], cfg.col_factors, cfg.table_rows[t])
        o = off[t * B:(t + 1) * B + 1]
        w = torch.as_tensor(psw[o[0]:o[-1]], dtype=torch.float64) if weighted else None
        ref = torch.nn.functional.embedding_bag(torch.as_tensor(idx[o[0]:o[-1]]), Wt,
                                                torch.as_tensor(o[:-1] - o[0]), mode=mode,
                                                per_sample_weights=w)
        np.testing.assert_allclose(out[:, t, :], ref.detach().numpy(), rtol=1e-12, atol=1e-13)
        (ref * torch.as_tensor(go[:, t, :], dtype=torch.float64)).sum().backward()
        for k in range(3):
            np.testing.assert_allclose(grads[t][k], ct[k].grad.numpy(), rtol=1e-11, atol=1e-12)


def test_weights_with_mean_rejected():
    orc = Oracle([10], [(2, 2, 3)], (1, 1, 2), 2)
    cores = [(np.ones((2, 1, 2), np.float32), np.ones((2, 2, 1, 2), np.float32), np.ones((3, 2, 2), np.float32))]
    with pytest.raises(OracleError) as e:
        orc.forward(cores, np.array([1]), np.array([0, 1]), 1, per_sample_weights=np.ones(1), mode="mean")
    assert e.value.code == ERR_INVALID


# ---------------------------------------------------------------------------
# Hybrid placement: small tables stay plain EmbeddingBag tables
# ---------------------------------------------------------------------------
def _hybrid_cfg():
    base = W.small_config([37, 300, 5, 1000], [(3, 4, 4), (7, 7, 7), (1, 2, 3), (10, 10, 10)],
                          (2, 3, 2), 4, 24, 1, 1.05)
    return W.hybrid(base, threshold=100)            # tables 0 and 2 dense, 1 and 3 TT


def test_hybrid_forward_and_gradients_match_torch():
    """Dense tables are plain nn.EmbeddingBag tables (W[M][N]); TT tables as before.  Forward and
    gradients (dW and dC_k) against torch embedding_bag + autograd on W / the materialised table."""
    cfg = _hybrid_cfg()
    assert cfg.dense == (True, False, True, False)
    rng = np.random.default_rng(21)
    T, B = cfg.num_tables, cfg.batch
    lens = rng.integers(0, 5, size=T * B); lens[1] = 0
    idx, off = W.make_batch(cfg, step=2, seed=21, lengths=lens)
    cores = W.make_cores(cfg, seed=21)
    go = W.make_grad_out(cfg, B, seed=21)
    orc = Oracle.from_config(cfg)
    out = orc.forward(cores, idx, off, B)
    grads = orc.backward(cores, idx, off, B, go)
    for t in range(T):
        o = off[t * B:(t + 1) * B + 1]
        if cfg.dense[t]:
            params = [torch.tensor(cores[t][0], dtype=torch.float64, requires_grad=True)]
            Wt = params[0]
        else:
            params = [torch.tensor(x, dtype=torch.float64, requires_grad=True) for x in cores[t]]
            Wt = materialise_torch(params, cfg.row_factors[t], cfg.col_factors, cfg.table_rows[t])
        ref = torch.nn.functional.embedding_bag(torch.as_tensor(idx[o[0]:o[-1]]), Wt,
                                                torch.as_tensor(o[:-1] - o[0]), mode="sum")
        np.testing.assert_allclose(out[:, t, :], ref.detach().numpy(), rtol=1e-12, atol=1e-13)
        (ref * torch.as_tensor(go[:, t, :], dtype=torch.float64)).sum().backward()
        for k, prm in enumerate(params):
            np.testing.assert_allclose(grads[t][k], prm.grad.numpy(), rtol=1e-11, atol=1e-12)
        if cfg.dense[t]:
            assert grads[t][1].size == 0 and grads[t][2].size == 0


def test_hybrid_plan_keys_tt_tables_first():
    """Plan keys number the TT tables first, then the dense tables (row id order); dense rows have
    no prefix (row_pfx = 0xFFFFFFFF) and the prefix rows end where the dense rows begin."""
    cfg = _hybrid_cfg()
    B = cfg.batch
    idx, off = W.make_batch(cfg, step=3, seed=22)
    orc = Oracle.from_config(cfg)
    plan = orc.plan(idx, off, B)
    T = cfg.num_tables
    mf = np.array(cfg.row_factors, np.int64)
    span = np.where(np.array(cfg.dense), np.array(cfg.table_rows), mf.prod(axis=1))
    order_t = [t for t in range(T) if not cfg.dense[t]] + [t for t in range(T) if cfg.dense[t]]
    base = np.zeros(T, np.int64)
    acc = 0
    for t in order_t:
        base[t] = acc
        acc += span[t]
    bag = np.repeat(np.arange(T * B), np.diff(off))
    tab = bag // B
    key = np.empty(len(idx), np.int64)
    for j, (i, t) in enumerate(zip(idx, tab)):
        if cfg.dense[t]:
            key[j] = base[t] + i
        else:
            d1, d2, d3 = np.unravel_index(i, tuple(mf[t]))
            key[j] = base[t] + (d2 * mf[t, 0] + d1) * mf[t, 2] + d3
    order = np.argsort(key, kind="stable")
    np.testing.assert_array_equal(plan["skey"], key[order])
    uk = np.unique(key)
    np.testing.assert_array_equal(plan["ukey"], uk)
    ntt = int(np.sum(uk < sum(span[t] for t in range(T) if not cfg.dense[t])))
    assert np.all(plan["row_pfx"][ntt:] == 0xFFFFFFFF) and np.all(plan["row_pfx"][:ntt] < plan["P"])
    assert plan["row_seg"][-1] == ntt
    assert set(plan["pfx_t"].tolist()) <= {1, 3}
