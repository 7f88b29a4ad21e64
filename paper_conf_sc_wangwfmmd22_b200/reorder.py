"""Offline index-bijection generator (Sec. IV) for ttemb_set_bijection.

The paper reorders *indices*, not table rows: an offline pass over sample batches builds a
bijection index_t(.) per table and every later lookup uses New_Batch = {index(i_j)};
that runtime gather runs inside libttemb's key-build kernel.  This module is the offline half
(host numpy, not on the training step -- "the generation of indexed bijections can be done
offline, so it will not bring additional overhead to the training process at runtime"):

  Alg. 2 lines 1-4 (global information): sort the ids by access frequency in descending order
  (Fre_order), take Hot_thre = Table_length * Hot_ratio, and give the hot ids (frequency rank <
  Hot_thre) the new ids 0 .. Hot_thre-1 in frequency order, "to gather hot embeddings
  together".
  The non-hot ids are the vertices of the paper's index graph (Alg. 2 lines 2-6): two ids that
  appear in the same batch are joined by an edge ("Batch_edges = Fre_batch.self_combinations()").
  `community_bijection` partitions that graph by modularity (refs [34]-[36]: the Louvain
  method, `louvain` below) and gives every community a contiguous block of new ids after the hot
  block ("assigning continuous indices to the vertices in the same community");
  `frequency_bijection` is the frequency-only variant (every non-hot id its own community).
  Readings (R26, R30): a "batch" of Alg. 2 is a window of `window` consecutive ids of
  one table's stream (all pairs of a 16 K-id batch would be 10^8 edges per batch); hot ids do not
  enter the graph (line 4's clamp would merge them into one vertex); edges are weighted by how
  many windows hold the pair; Q = (1/2m) sum_ij [A_ij - k_i k_j / 2m] delta(c_i, c_j) (P:277's
  formula is garbled, this is the modularity of its ref [36]).

Ties in frequency are broken by the smaller old id, so the result is deterministic.
"""
from __future__ import annotations

from typing import Dict, Iterable, List, Optional, Sequence, Tuple

import numpy as np


def table_ids(indices: np.ndarray, offsets: np.ndarray, num_tables: int, batch: int) -> List[np.ndarray]:
    """Split a table-major batch (offsets[T*B+1]) into the id stream of each table."""
    off = np.asarray(offsets, dtype=np.int64)
    idx = np.asarray(indices, dtype=np.int64)
    return [idx[off[t * batch]:off[(t + 1) * batch]] for t in range(num_tables)]


def frequency_order(counts: np.ndarray) -> np.ndarray:
    """Fre_order (Alg. 2 input): rank[i] = position of id i when sorted by (count desc, id asc)."""
    M = len(counts)
    order = np.lexsort((np.arange(M), -np.asarray(counts, dtype=np.int64)))
    rank = np.empty(M, dtype=np.int64)
    rank[order] = np.arange(M)
    return rank


def table_bijection(counts: np.ndarray, hot_ratio: Optional[float] = None) -> np.ndarray:
    """index_t for one table: new id of every old id (a permutation of [0, M)).

    hot_ratio=None takes every id seen in the sample as hot (Hot_thre = #ids with count > 0)."""
    counts = np.asarray(counts, dtype=np.int64)
    M = len(counts)
    rank = frequency_order(counts)
    if hot_ratio is None:
        hot = int(np.count_nonzero(counts))
    else:
        hot = int(min(M, max(0, int(M * float(hot_ratio)))))    # Hot_thre = Table_length * Hot_ratio
    new = np.empty(M, dtype=np.int64)
    is_hot = rank < hot
    new[is_hot] = rank[is_hot]
    cold = np.flatnonzero(~is_hot)                               # ascending old id
    new[cold] = hot + np.arange(len(cold))
    return new


def frequency_bijection(table_rows: Sequence[int], batches: Iterable[Tuple[np.ndarray, np.ndarray, int]],
                        hot_ratio: Optional[float] = None) -> np.ndarray:
    """Concatenated bijection for ttemb_set_bijection (uint32 [sum M_t], table t at M_0+..+M_{t-1}).

    batches: (indices, offsets, batch) sample batches of the training stream (raw ids)."""
    T = len(table_rows)
    counts = [np.zeros(int(M), dtype=np.int64) for M in table_rows]
    for idx, off, B in batches:
        for t, ids in enumerate(table_ids(idx, off, T, B)):
            if len(ids):
                if ids.min() < 0 or ids.max() >= table_rows[t]:
                    raise ValueError(f"id out of range in table {t}")
                counts[t] += np.bincount(ids, minlength=int(table_rows[t]))
    maps = [table_bijection(c, hot_ratio) for c in counts]
    return np.concatenate(maps).astype(np.uint32) if maps else np.zeros(0, np.uint32)


def split_bijection(bij: np.ndarray, table_rows: Sequence[int]) -> List[np.ndarray]:
    """Per-table views of a concatenated bijection."""
    out, o = [], 0
    for M in table_rows:
        out.append(np.asarray(bij[o:o + int(M)]))
        o += int(M)
    return out


# ---------------------------------------------------------------------------
# Alg. 2 index graph + modularity communities
# ---------------------------------------------------------------------------
def index_graph(streams: Iterable[np.ndarray], rank: np.ndarray, hot: int, window: int = 32
                ) -> Tuple[int, np.ndarray, np.ndarray, np.ndarray]:
    """Alg. 2 for one table: vertices = non-hot ids (vertex = frequency rank - Hot_thre), an
    edge (weight 1 per window) between every two distinct non-hot ids of a window.
    Returns (n_vertices, u, v, w) with u < v, merged duplicates."""
    n = len(rank) - hot
    keys: Dict[int, int] = {}
    for ids in streams:
        fre = np.asarray(rank)[np.asarray(ids, dtype=np.int64)]          # line 3: Fre_order[Batch]
        for s0 in range(0, len(fre), window):
            b = np.unique(fre[s0:s0 + window])
            b = b[b >= hot] - hot                                          # line 4: non-hot only
            if len(b) < 2:
                continue
            iu, ju = np.triu_indices(len(b), 1)                            # line 5: self_combinations
            for k in (b[iu] * n + b[ju]).tolist():
                keys[k] = keys.get(k, 0) + 1
    if not keys:
        z = np.zeros(0, np.int64)
        return n, z, z, np.zeros(0, np.float64)
    k = np.fromiter(keys.keys(), np.int64, len(keys))
    w = np.fromiter(keys.values(), np.float64, len(keys))
    return n, k // n, k % n, w


def modularity(n: int, u: np.ndarray, v: np.ndarray, w: np.ndarray, comm: np.ndarray) -> float:
    """Newman modularity (ref [36]) of an undirected weighted graph (edges u-v once each):
    Q = sum_c [ L_c / m - (d_c / 2m)^2 ], L_c the weight inside c, d_c its total degree."""
    m = float(np.sum(w))
    if m == 0.0:
        return 0.0
    comm = np.asarray(comm)
    deg = np.bincount(u, weights=w, minlength=n) + np.bincount(v, weights=w, minlength=n)
    nc = int(comm.max()) + 1 if len(comm) else 0
    inside = comm[u] == comm[v]
    lc = np.bincount(comm[u][inside], weights=w[inside], minlength=nc)
    dc = np.bincount(comm, weights=deg, minlength=nc)
    return float(np.sum(lc / m - (dc / (2.0 * m)) ** 2))


def _csr(n, u, v, w):
    """Symmetric adjacency (both directions; a self-loop once with weight 2w)."""
    loop = u == v
    src = np.concatenate([u[~loop], v[~loop], u[loop]])
    dst = np.concatenate([v[~loop], u[~loop], v[loop]])
    wt = np.concatenate([w[~loop], w[~loop], 2.0 * w[loop]])
    order = np.argsort(src, kind="stable")
    src, dst, wt = src[order], dst[order], wt[order]
    ptr = np.zeros(n + 1, np.int64)
    np.add.at(ptr, src + 1, 1)
    return np.cumsum(ptr), dst, wt


def louvain(n: int, u: np.ndarray, v: np.ndarray, w: np.ndarray) -> np.ndarray:
    """Louvain communities by the native implementation in libttemb.so (ttemb_louvain, the same
    algorithm as `louvain_py`, which the tests compare it with)."""
    import ctypes as C
    from paper_conf_sc_wangwfmmd22_b200 import _lib as L
    u = np.ascontiguousarray(u, np.int64)
    v = np.ascontiguousarray(v, np.int64)
    w = np.ascontiguousarray(w, np.float64)
    lab = np.zeros(max(n, 1), np.int64)
    p64 = C.POINTER(C.c_int64)
    rc = L.load().ttemb_louvain(int(n), len(u), u.ctypes.data_as(p64), v.ctypes.data_as(p64),
                                w.ctypes.data_as(C.POINTER(C.c_double)), lab.ctypes.data_as(p64))
    L.check(rc, "ttemb_louvain")
    return lab[:n]


def louvain_py(n: int, u: np.ndarray, v: np.ndarray, w: np.ndarray, max_levels: int = 16,
               max_passes: int = 32) -> np.ndarray:
    """Modularity maximisation by the Louvain method (refs [34], [35] of the paper): local moves
    of single vertices to the neighbouring community with the largest modularity gain
    dQ ~ k_i,in(C) - tot(C) k_i / 2m (vertices in index order, ties to the smaller community),
    then aggregation of communities into vertices, until no move improves Q.  Deterministic.
    Returns a community label per vertex (0 .. C-1, ordered by first vertex)."""
    labels = np.arange(n, dtype=np.int64)
    cu, cv, cw = np.asarray(u, np.int64), np.asarray(v, np.int64), np.asarray(w, np.float64)
    cn = n
    for _ in range(max_levels):
        if len(cw) == 0:
            break
        ptr, dst, wt = _csr(cn, cu, cv, cw)
        k = np.zeros(cn)
        np.add.at(k, np.repeat(np.arange(cn), np.diff(ptr)), wt)
        m2 = float(k.sum())
        comm = np.arange(cn, dtype=np.int64)
        tot = k.copy()
        improved = False
        for _ in range(max_passes):
            moved = 0
            for i in range(cn):
                a, b = ptr[i], ptr[i + 1]
                nb, nw = dst[a:b], wt[a:b]
                keep = nb != i
                nb, nw = nb[keep], nw[keep]
                ci = comm[i]
                tot[ci] -= k[i]
                kin: Dict[int, float] = {}
                for c, x in zip(comm[nb].tolist(), nw.tolist()):
                    kin[c] = kin.get(c, 0.0) + x
                best, best_gain = ci, kin.get(ci, 0.0) - tot[ci] * k[i] / m2
                for c in sorted(kin):
                    gain = kin[c] - tot[c] * k[i] / m2
                    if gain > best_gain + 1e-12:
                        best, best_gain = c, gain
                tot[best] += k[i]
                if best != ci:
                    comm[i] = best
                    moved += 1
            if moved == 0:
                break
            improved = True
        if not improved:
            break
        _, comm = np.unique(comm, return_inverse=True)
        labels = comm[labels]
        cn = int(comm.max()) + 1
        lo = np.minimum(comm[cu], comm[cv]) * cn + np.maximum(comm[cu], comm[cv])
        uk, inv = np.unique(lo, return_inverse=True)
        cw = np.bincount(inv, weights=cw)
        cu, cv = uk // cn, uk % cn
    # labels numbered by first occurrence
    _, first = np.unique(labels, return_index=True)
    order = np.argsort(first)
    remap = np.empty(len(order), np.int64)
    remap[order] = np.arange(len(order))
    return remap[labels] if n else labels


def table_community_bijection(counts: np.ndarray, streams: Sequence[np.ndarray],
                              hot_ratio: float, window: int = 32) -> np.ndarray:
    """index_t for one table with communities: hot ids (frequency rank < Hot_thre)
    get new ids 0 .. Hot_thre-1 in frequency order; the non-hot ids of the index graph follow
    community by community (communities ordered by total access count, descending; ids inside
    a community by frequency rank); ids outside the graph come last in frequency-rank order."""
    counts = np.asarray(counts, dtype=np.int64)
    M = len(counts)
    rank = frequency_order(counts)
    hot = int(min(M, max(0, int(M * float(hot_ratio)))))
    n, u, v, w = index_graph(streams, rank, hot, window)
    comm = louvain(n, u, v, w)
    by_rank = np.argsort(rank)                        # old id of every frequency rank
    in_graph = np.zeros(n, bool)
    in_graph[u] = True
    in_graph[v] = True
    new = np.empty(M, np.int64)
    new[by_rank[:hot]] = np.arange(hot)
    verts = np.flatnonzero(in_graph)
    csum = np.bincount(comm[verts], weights=counts[by_rank[hot + verts]], minlength=int(comm.max()) + 1 if n else 0)
    # communities by total access count (descending, ties by label); inside one, by frequency rank
    crank = np.empty(len(csum), np.int64)
    corder = np.lexsort((np.arange(len(csum)), -csum))
    crank[corder] = np.arange(len(csum))
    seq = verts[np.lexsort((verts, crank[comm[verts]]))]
    nxt = hot
    new[by_rank[hot + seq]] = nxt + np.arange(len(seq))
    nxt += len(seq)
    rest = np.flatnonzero(~in_graph)
    new[by_rank[hot + rest]] = nxt + np.arange(len(rest))
    return new


def community_bijection(table_rows: Sequence[int], batches: Iterable[Tuple[np.ndarray, np.ndarray, int]],
                        hot_ratio: float = 0.0, window: int = 32) -> np.ndarray:
    """Concatenated bijection (ttemb_set_bijection layout) from the full generator of Sec. IV-C:
    frequency order (global information) + index graph communities (local information)."""
    T = len(table_rows)
    counts = [np.zeros(int(M), dtype=np.int64) for M in table_rows]
    streams: List[List[np.ndarray]] = [[] for _ in range(T)]
    for idx, off, B in batches:
        for t, ids in enumerate(table_ids(idx, off, T, B)):
            if len(ids):
                if ids.min() < 0 or ids.max() >= table_rows[t]:
                    raise ValueError(f"id out of range in table {t}")
                counts[t] += np.bincount(ids, minlength=int(table_rows[t]))
                streams[t].append(ids)
    maps = [table_community_bijection(counts[t], streams[t], hot_ratio, window) for t in range(T)]
    return np.concatenate(maps).astype(np.uint32) if maps else np.zeros(0, np.uint32)
