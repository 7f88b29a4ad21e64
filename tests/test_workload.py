"""Seeded generator checks (synth/workload.py; no method arithmetic)."""
import numpy as np

from synth import workload as W


def test_near_cubic_rule_examples():
    # DESIGN.md R11 worked values
    assert W.near_cubic(9_000_000) == (207, 209, 209)
    assert W.near_cubic(10_131_227) == (216, 217, 217)
    assert W.near_cubic(40_000_000) == (342, 342, 342)
    assert W.near_cubic(3) == (1, 2, 2)
    for m in [1, 2, 4, 7, 8, 9, 26, 1000, 39884406]:
        f = W.near_cubic(m)
        assert f[0] * f[1] * f[2] >= m


def test_configs_shapes():
    c4 = W.config("c4")
    assert c4.num_tables == 26 and c4.dim == 64 and c4.rank == 64 and c4.batch == 16384
    assert max(c4.table_rows) <= 40_000_000
    c5 = W.config("c5", 128)
    assert c5.num_tables == 8 and c5.dim == 128 and c5.pooling == 20
    assert W.config("c1").row_factors == ((10, 10, 10),)


def test_batch_is_seeded_and_in_range():
    cfg = W.config("c2")
    i1, o1 = W.make_batch(cfg, step=3, seed=9, batch=256)
    i2, o2 = W.make_batch(cfg, step=3, seed=9, batch=256)
    np.testing.assert_array_equal(i1, i2)
    np.testing.assert_array_equal(o1, o2)
    B = 256
    for t in range(cfg.num_tables):
        ids = i1[o1[t * B]:o1[(t + 1) * B]]
        assert ids.min() >= 0 and ids.max() < cfg.table_rows[t]
    i3, _ = W.make_batch(cfg, step=4, seed=9, batch=256)
    assert not np.array_equal(i1, i3)


def test_zipf_skew_identity_map():
    g = W.rng("t")
    ids = W.zipf_ids(g, 1_000_000, 1.05, 200_000)
    # rank-1 id (0) is the most frequent; U/n well below 1
    assert np.bincount(ids[ids < 10]).argmax() == 0
    assert len(np.unique(ids)) / len(ids) < 0.6


def test_shard_batch_partitions_samples():
    cfg = W.small_config([50, 60], [(5, 5, 2), (4, 4, 4)], (1, 1, 2), 2, 8, 3)
    idx, off = W.make_batch(cfg, seed=1)
    parts = [W.shard_batch(idx, off, 2, 8, r, 4) for r in range(4)]
    assert sum(len(p[0]) for p in parts) == len(idx)
    for r, (i, o, bl) in enumerate(parts):
        assert bl == 2 and o[0] == 0 and o[-1] == len(i)
