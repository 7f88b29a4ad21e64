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


# ---------------------------------------------------------------------------
# Alg. 2 index graph + modularity communities
# ---------------------------------------------------------------------------
def _nx_partition(comm):
    groups = {}
    for i, c in enumerate(comm):
        groups.setdefault(int(c), set()).add(i)
    return list(groups.values())


def test_modularity_matches_networkx():
    """The modularity of ref [36] (our reading of the garbled P:277 formula) equals networkx's
    implementation on random weighted graphs and partitions."""
    nx = pytest.importorskip("networkx")
    rng = np.random.default_rng(0)
    for _ in range(5):
        n = 30
        e = {(int(a), int(b)) for a, b in rng.integers(0, n, size=(80, 2)) if a < b}
        u = np.array([a for a, b in e]); v = np.array([b for a, b in e])
        w = rng.integers(1, 4, size=len(u)).astype(float)
        comm = rng.integers(0, 4, size=n)
        G = nx.Graph()
        G.add_nodes_from(range(n))
        G.add_weighted_edges_from(zip(u.tolist(), v.tolist(), w.tolist()))
        ref = nx.algorithms.community.modularity(G, _nx_partition(comm), weight="weight")
        assert abs(R.modularity(n, u, v, w, comm) - ref) < 1e-12


def test_louvain_recovers_planted_communities():
    """Two 6-cliques joined by one edge: Louvain puts each clique in one community, and its
    modularity is at least networkx's Louvain result on the same graph."""
    nx = pytest.importorskip("networkx")
    edges = [(a, b) for a in range(6) for b in range(a + 1, 6)]
    edges += [(a + 6, b + 6) for a, b in edges] + [(5, 6)]
    u = np.array([a for a, b in edges]); v = np.array([b for a, b in edges]); w = np.ones(len(edges))
    comm = R.louvain(12, u, v, w)
    assert len(set(comm[:6].tolist())) == 1 and len(set(comm[6:].tolist())) == 1 and comm[0] != comm[6]
    G = nx.Graph()
    G.add_edges_from(edges)
    ref = nx.algorithms.community.modularity(G, nx.algorithms.community.louvain_communities(G, seed=0))
    assert R.modularity(12, u, v, w, comm) >= ref - 1e-12


def test_louvain_never_below_singletons_and_is_deterministic():
    rng = np.random.default_rng(1)
    n = 60
    e = {(int(a), int(b)) for a, b in rng.integers(0, n, size=(200, 2)) if a < b}
    u = np.array([a for a, b in e]); v = np.array([b for a, b in e]); w = np.ones(len(u))
    c1 = R.louvain(n, u, v, w)
    assert R.modularity(n, u, v, w, c1) >= R.modularity(n, u, v, w, np.arange(n))
    np.testing.assert_array_equal(c1, R.louvain(n, u, v, w))


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_native_louvain_equals_python_reference(seed):
    """ttemb_louvain (C++ in libttemb.so) and the plain Python Louvain give the same labels on
    random weighted graphs (integer weights: every sum is exact, so the moves are identical)."""
    rng = np.random.default_rng(seed)
    n = 80
    e = {(int(a), int(b)) for a, b in rng.integers(0, n, size=(300, 2)) if a < b}
    u = np.array([a for a, b in e]); v = np.array([b for a, b in e])
    w = rng.integers(1, 5, size=len(u)).astype(float)
    np.testing.assert_array_equal(R.louvain(n, u, v, w), R.louvain_py(n, u, v, w))


def test_index_graph_follows_alg2():
    """Alg. 2: per window, all pairs of distinct NON-hot ids (frequency rank >= Hot_thre) become
    edges (vertex = rank - Hot_thre); repeated pairs add weight; hot ids never enter."""
    rank = np.array([0, 1, 2, 3, 4, 5])          # id i has frequency rank i
    n, u, v, w = R.index_graph([np.array([0, 3, 4, 3, 5, 1])], rank, hot=2, window=3)
    # windows [0,3,4] -> non-hot {3,4} -> (1,2); [3,5,1] -> {3,5} -> (1,3)
    assert n == 4
    got = sorted(zip(u.tolist(), v.tolist(), w.tolist()))
    assert got == [(1, 2, 1.0), (1, 3, 1.0)]
    n, u, v, w = R.index_graph([np.array([3, 4, 3, 4])], rank, hot=2, window=2)
    assert sorted(zip(u.tolist(), v.tolist(), w.tolist())) == [(1, 2, 2.0)]


def test_community_bijection_clusters_session_topics():
    """On a stream with local information (W.make_session_batch: each batch concentrates on a
    topic's id set, scattered over the raw id space), the community bijection is a permutation
    per table that keeps the hot block, and it packs each topic into few prefixes: the mean
    number of distinct prefixes (id // m3, Alg. 1's Buf_idx) per batch drops below the
    frequency-only bijection's and the raw ids'."""
    cfg = W.small_config([50000], [(37, 37, 37)], (2, 2, 2), 4, 512, 1, 1.05).replace(id_map="perm")
    kw = dict(topics=4, topic_frac=0.6, topic_size=300)
    hist = [W.make_session_batch(cfg, step=s, seed=1, **kw) + (cfg.batch,) for s in range(8)]
    bij_c = R.community_bijection(cfg.table_rows, hist, hot_ratio=0.001, window=32)
    bij_f = R.frequency_bijection(cfg.table_rows, hist, hot_ratio=0.001)
    M = cfg.table_rows[0]
    assert np.array_equal(np.sort(bij_c.astype(np.int64)), np.arange(M))
    m3 = cfg.row_factors[0][2]
    ev = [W.make_session_batch(cfg, step=s, seed=2, **kw)[0] for s in range(8, 12)]
    p_raw = np.mean([len(np.unique(b // m3)) for b in ev])
    p_freq = np.mean([len(np.unique(bij_f.astype(np.int64)[b] // m3)) for b in ev])
    p_comm = np.mean([len(np.unique(bij_c.astype(np.int64)[b] // m3)) for b in ev])
    assert p_comm < p_freq <= p_raw, (p_raw, p_freq, p_comm)
