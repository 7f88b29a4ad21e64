"""Offline index-bijection generator (paper_conf_sc_wangwfmmd22_b200/reorder.py; Alg. 2 lines 1-4,
P:204-277).  Host-only logic (numpy), no GPU: the generator's properties, and that the bijection
restores prefix reuse on a raw-id (permuted) Zipf stream, counted with the oracle's plan."""
import numpy as np
import pytest

from oracle import Oracle
from synth import workload as W

import importlib.util, os   # noqa: E401,E402  (by path: the package __init__ needs the built .so)
_p = os.path.join(os.path.dirname(os.path.dirname(__file__)), "paper_conf_sc_wangwfmmd22_b200", "reorder.py")
_s = importlib.util.spec_from_file_location("_reorder", _p)
R = importlib.util.module_from_spec(_s)
_s.loader.exec_module(R)


def test_frequency_order_and_hot_block():
    counts = np.array([0, 5, 2, 5, 0, 9, 1])
    rank = R.frequency_order(counts)
    # (count desc, id asc): 5(9), 1(5), 3(5), 2(2), 6(1), 0(0), 4(0)
    assert list(np.argsort(rank)) == [5, 1, 3, 2, 6, 0, 4]
    new = R.table_bijection(counts)                 # hot = the 5 ids seen
    assert sorted(new) == list(range(7))
    assert list(new[[5, 1, 3, 2, 6]]) == [0, 1, 2, 3, 4]
    assert list(new[[0, 4]]) == [5, 6]              # cold ids keep their order after the hot block
    new2 = R.table_bijection(counts, hot_ratio=2 / 7)   # Hot_thre = Table_length * Hot_ratio = 2
    assert list(new2[[5, 1]]) == [0, 1] and list(new2[[0, 2, 3, 4, 6]]) == [2, 3, 4, 5, 6]


def test_bijection_is_a_permutation_per_table():
    cfg = W.small_config([37, 100, 5, 1000], [(3, 4, 4), (5, 4, 5), (1, 2, 3), (10, 10, 10)],
                         (2, 3, 2), 5, 64, 2, 1.05).replace(id_map="perm")
    batches = [W.make_batch(cfg, step=s, seed=1) + (cfg.batch,) for s in range(4)]
    bij = R.frequency_bijection(cfg.table_rows, batches)
    assert bij.dtype == np.uint32 and len(bij) == sum(cfg.table_rows)
    for M, m in zip(cfg.table_rows, R.split_bijection(bij, cfg.table_rows)):
        assert np.array_equal(np.sort(m), np.arange(M))


def test_bijection_restores_prefix_reuse_on_raw_ids():
    """with raw (permuted) ids the batch's indices are spread out and few TT prefixes
    are shared; the frequency bijection gathers the hot ids, so the unique-prefix count P of a
    later batch drops towards that of the clustered (identity) stream."""
    base = W.small_config([200000, 50000], [(59, 59, 58), (37, 37, 37)], (2, 2, 4), 8, 2048, 1, 1.05)
    raw = base.replace(id_map="perm")
    hist = [W.make_batch(raw, step=s, seed=3) + (raw.batch,) for s in range(1, 9)]
    bij = R.frequency_bijection(raw.table_rows, hist)
    orc = Oracle.from_config(raw)
    idx, off = W.make_batch(raw, step=0, seed=3)
    p_raw = orc.plan(idx, off, raw.batch)["P"]
    p_bij = orc.plan(orc.apply_bijection(R.split_bijection(bij, raw.table_rows), idx, off, raw.batch),
                     off, raw.batch)["P"]
    ii, oi = W.make_batch(base, step=0, seed=3)
    p_id = orc.plan(ii, oi, base.batch)["P"]
    assert p_bij < 0.8 * p_raw, (p_raw, p_bij, p_id)
    assert p_bij <= 1.5 * p_id, (p_raw, p_bij, p_id)
