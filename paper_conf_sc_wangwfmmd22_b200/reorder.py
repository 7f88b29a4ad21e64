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
  The non-hot ids are the vertices of the paper's index graph, which is partitioned by
  modularity-based community detection.  That step is not built here (SURVEY.md 8(f2):
  "community detection after that"): the non-hot ids keep their relative order, i.e. every one
  is its own community, numbered after the hot block in ascending old id.

Ties in frequency are broken by the smaller old id, so the result is deterministic.
"""
from __future__ import annotations

from typing import Iterable, List, Optional, Sequence, Tuple

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
