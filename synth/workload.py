"""Seeded synthetic workloads for the TT-EmbeddingBag hot path.

This module is shared by the CPU oracle tests, the CUDA parity tests and
bench.py.  It holds NONE of the method's arithmetic (no TT digits, no
contraction, no pooling): only table shapes, factor choices, id streams,
offsets, core initialisation and output gradients, all drawn from seeded
numpy generators.

Paper context (PAPER.md, cited as P:<line>):
  * access skew: "the distribution of activated sparse indices follows a
    power-law distribution" (Sec. II-C) -> bounded Zipf(s) ids;
  * after the paper's bijection reordering hot ids are clustered
    (Alg. 2) -> primary id map "identity" (Zipf rank r
    -> id r-1); secondary "perm" (seeded permutation, raw ids);
  * "initialized randomly" -> seeded uniform cores (R21);
  * factorisation M <= m1*m2*m3, N = n1*n2*n3 (Eq. 2); the factor
    choice for the synthetic configs is the near-cubic rule (R11).

The five BASELINE.json configs are reproduced by `config(name)`.
"""
from __future__ import annotations

import dataclasses
import functools
import hashlib
from typing import List, Optional, Sequence, Tuple

import numpy as np

# ---------------------------------------------------------------------------
# Table-size profiles (the Kaggle / Terabyte lists are the
# public DLRM preprocessing cardinalities, used only as a size profile; the
# Avazu list is invented to match "largest ~9M").
# ---------------------------------------------------------------------------
AVAZU_ROWS = [9_000_000, 2_700_000, 8_600, 8_300, 7_800, 4_800, 2_700, 560, 440, 240,
              170, 70, 60, 36, 26, 9, 8, 7, 5, 4]
KAGGLE_ROWS = [1460, 583, 10131227, 2202608, 305, 24, 12517, 633, 3, 93145, 5683,
               8351593, 3194, 27, 14992, 5461306, 10, 5652, 2173, 4, 7046547, 18, 15,
               286181, 105, 142572]
TB_ROWS = [39884406, 39043, 17289, 7420, 20263, 3, 7120, 1543, 63, 38532951, 2953546,
           403346, 10, 2208, 11938, 155, 4, 976, 14, 39979771, 25641295, 39664984,
           585935, 12972, 108, 36]


def icbrt_ceil(m: int) -> int:
    """Smallest integer c with c**3 >= m (exact integer arithmetic)."""
    c = max(1, int(round(m ** (1.0 / 3.0))))
    while c ** 3 < m:
        c += 1
    while c > 1 and (c - 1) ** 3 >= m:
        c -= 1
    return c


def near_cubic(m: int) -> Tuple[int, int, int]:
    """Near-cubic row factorisation (reading R11).

    Start from c = ceil(M^(1/3)) for all three factors, then shrink m1, then
    m2, one step at a time while the product stays >= M.
    9_000_000 -> (207, 209, 209); 40_000_000 -> (342, 342, 342); 3 -> (1, 2, 2).
    """
    if m < 1:
        raise ValueError("table needs at least one row")
    c = icbrt_ceil(m)
    f = [c, c, c]
    for k in (0, 1):
        while f[k] > 1 and (f[k] - 1) * f[(k + 1) % 3] * f[(k + 2) % 3] >= m:
            f[k] -= 1
    return (f[0], f[1], f[2])


@dataclasses.dataclass(frozen=True)
class TTConfig:
    name: str
    table_rows: Tuple[int, ...]
    row_factors: Tuple[Tuple[int, int, int], ...]
    col_factors: Tuple[int, int, int]
    rank: int
    batch: int                      # global batch (samples)
    pooling: int                    # fixed bag length L (ids per bag)
    zipf_s: Optional[float]         # None -> uniform ids
    id_map: str = "identity"        # "identity" | "perm"
    dense: Tuple[bool, ...] = ()    # hybrid placement: table kept uncompressed; () = all TT

    def is_dense(self, t: int) -> bool:
        return bool(self.dense) and bool(self.dense[t])

    @property
    def num_tables(self) -> int:
        return len(self.table_rows)

    @property
    def dim(self) -> int:
        n1, n2, n3 = self.col_factors
        return n1 * n2 * n3

    def lookups_per_step(self, batch: Optional[int] = None) -> int:
        return (self.batch if batch is None else batch) * self.num_tables * self.pooling

    def replace(self, **kw) -> "TTConfig":
        return dataclasses.replace(self, **kw)


def _mk(name, rows, col, rank, batch, pooling, zipf_s, factors=None, id_map="identity"):
    rows = tuple(int(r) for r in rows)
    if factors is None:
        factors = tuple(near_cubic(r) for r in rows)
    return TTConfig(name, rows, tuple(tuple(f) for f in factors), tuple(col), int(rank),
                    int(batch), int(pooling), zipf_s, id_map)


def config(name: str, rank: Optional[int] = None) -> TTConfig:
    """The five BASELINE.json configs ("c1".."c5"); c5 takes rank 32/64/128."""
    name = name.lower()
    if name == "c1":
        return _mk("c1-tiny", [1000], (2, 2, 4), 8, 64, 1, None, factors=[(10, 10, 10)])
    if name == "c2":
        return _mk("c2-avazu", AVAZU_ROWS, (2, 2, 4), 16, 4096, 1, 1.05)
    if name == "c3":
        return _mk("c3-kaggle", KAGGLE_ROWS, (2, 2, 4), 32, 8192, 1, 1.05)
    if name == "c4":
        return _mk("c4-terabyte", TB_ROWS, (4, 4, 4), 64, 16384, 1, 1.05)
    if name == "c5":
        r = 64 if rank is None else int(rank)
        if r not in (32, 64, 128):
            raise ValueError("c5 rank must be 32, 64 or 128")
        return _mk(f"c5-multihot-r{r}", [40_000_000] * 8, (4, 4, 8), r, 65536, 20, 1.05)
    raise KeyError(name)


ALL_CONFIGS = ("c1", "c2", "c3", "c4", "c5")

HYBRID_THRESHOLD = 1_000_000   # "decompose the embedding tables that have more than 1 million rows"


def hybrid(cfg: TTConfig, threshold: int = HYBRID_THRESHOLD) -> TTConfig:
    """The paper's end-to-end placement: tables with more than `threshold` rows are TT
    compressed, the others stay plain (dense) EmbeddingBag tables."""
    return cfg.replace(name=cfg.name + "-hybrid", dense=tuple(M <= threshold for M in cfg.table_rows))


# ---------------------------------------------------------------------------
# Seeds
# ---------------------------------------------------------------------------
def _seed(*parts) -> np.random.SeedSequence:
    h = hashlib.sha256("/".join(str(p) for p in parts).encode()).digest()
    return np.random.SeedSequence(int.from_bytes(h[:16], "little"))


def rng(*parts) -> np.random.Generator:
    return np.random.Generator(np.random.PCG64(_seed(*parts)))


# ---------------------------------------------------------------------------
# Id streams
# ---------------------------------------------------------------------------
@functools.lru_cache(maxsize=32)
def _zipf_cdf(m: int, s: float) -> np.ndarray:
    """Cumulative distribution of the bounded Zipf law p_r ~ r^-s, r = 1..m."""
    r = np.arange(1, m + 1, dtype=np.float64)
    w = r ** (-s)
    c = np.cumsum(w)
    c /= c[-1]
    return c


@functools.lru_cache(maxsize=32)
def _perm(m: int, seed_tag: str) -> np.ndarray:
    return rng("perm", seed_tag, m).permutation(m).astype(np.int64)


def zipf_ids(g: np.random.Generator, m: int, s: Optional[float], n: int,
             id_map: str = "identity", perm_tag: str = "") -> np.ndarray:
    """n ids in [0, m): exact bounded inverse-CDF Zipf (or uniform if s is None)."""
    if n == 0:
        return np.zeros(0, dtype=np.int64)
    if s is None:
        ids = g.integers(0, m, size=n, dtype=np.int64)
    else:
        u = g.random(n)
        ids = np.searchsorted(_zipf_cdf(m, float(s)), u, side="right").astype(np.int64)
        np.minimum(ids, m - 1, out=ids)        # guard u rounding to the last bin
    if id_map == "perm":
        ids = _perm(m, perm_tag)[ids]
    elif id_map != "identity":
        raise ValueError(id_map)
    return ids


def make_batch(cfg: TTConfig, step: int = 0, seed: int = 0, batch: Optional[int] = None,
               lengths: Optional[np.ndarray] = None) -> Tuple[np.ndarray, np.ndarray]:
    """Global batch: (indices int64 [nnz], offsets int64 [T*B+1]), table-major.

    Bag (t, b) = indices[offsets[t*B+b] : offsets[t*B+b+1]].
    `lengths` ([T*B] ints) overrides the fixed pooling factor (variable L,
    empty bags allowed).
    """
    B = cfg.batch if batch is None else int(batch)
    T = cfg.num_tables
    if lengths is None:
        lengths = np.full(T * B, cfg.pooling, dtype=np.int64)
    lengths = np.asarray(lengths, dtype=np.int64)
    assert lengths.shape == (T * B,)
    offsets = np.zeros(T * B + 1, dtype=np.int64)
    np.cumsum(lengths, out=offsets[1:])
    parts = []
    for t in range(T):
        n_t = int(offsets[(t + 1) * B] - offsets[t * B])
        g = rng("ids", cfg.name, cfg.id_map, seed, step, t)
        parts.append(zipf_ids(g, cfg.table_rows[t], cfg.zipf_s, n_t, cfg.id_map,
                              perm_tag=f"{cfg.name}/{t}"))
    indices = np.concatenate(parts) if parts else np.zeros(0, dtype=np.int64)
    return indices, offsets


def make_session_batch(cfg: TTConfig, step: int = 0, seed: int = 0, batch: Optional[int] = None,
                       topics: int = 8, topic_frac: float = 0.5, topic_size: int = 4096
                       ) -> Tuple[np.ndarray, np.ndarray]:
    """A stream with LOCAL information (a batch reflects the user behaviour of one
    period): batch `step` belongs to session topic k = step % topics; each id is, with
    probability topic_frac, uniform over topic k's fixed id set (topic_size ids of the table,
    disjoint across topics, scattered by the table's raw-id permutation), else a Zipf(s) id
    through the same permutation.  Used to measure the community part of the paper's index
    bijection (Alg. 2 + modularity communities); id generation only."""
    B = cfg.batch if batch is None else int(batch)
    T = cfg.num_tables
    lengths = np.full(T * B, cfg.pooling, dtype=np.int64)
    offsets = np.zeros(T * B + 1, dtype=np.int64)
    np.cumsum(lengths, out=offsets[1:])
    k = step % topics
    parts = []
    for t in range(T):
        m = cfg.table_rows[t]
        n_t = int(offsets[(t + 1) * B] - offsets[t * B])
        g = rng("session", cfg.name, seed, step, t)
        perm = _perm(m, f"{cfg.name}/{t}")
        ts = min(topic_size, max(1, m // (topics + 1)))
        ranks = zipf_ids(g, m, cfg.zipf_s, n_t, "identity")
        topic = g.random(n_t) < topic_frac
        # topic k's ids: ranks [m - (k + 1) ts, m - k ts) (the cold tail), permuted like every id
        ranks[topic] = m - (k + 1) * ts + g.integers(0, ts, size=int(topic.sum()))
        parts.append(perm[ranks])
    indices = np.concatenate(parts) if parts else np.zeros(0, dtype=np.int64)
    return indices, offsets


def shard_batch(indices: np.ndarray, offsets: np.ndarray, num_tables: int, batch: int,
                rank: int, world: int) -> Tuple[np.ndarray, np.ndarray, int]:
    """Rank `rank` of `world` takes samples [rank*B/G, (rank+1)*B/G) of every table
    (SURVEY 8(e)); returns its (indices, offsets rebased to 0, local batch)."""
    if batch % world:
        raise ValueError("global batch must divide by world size")
    bl = batch // world
    b0 = rank * bl
    T = num_tables
    idx_parts = []
    lens = []
    for t in range(T):
        s = int(offsets[t * batch + b0])
        e = int(offsets[t * batch + b0 + bl])
        idx_parts.append(indices[s:e])
        lens.append(np.diff(offsets[t * batch + b0: t * batch + b0 + bl + 1]))
    lens = np.concatenate(lens) if lens else np.zeros(0, np.int64)
    off = np.zeros(T * bl + 1, dtype=np.int64)
    np.cumsum(lens, out=off[1:])
    idx = np.concatenate(idx_parts) if idx_parts else np.zeros(0, np.int64)
    return idx, off, bl


# ---------------------------------------------------------------------------
# Parameters and upstream gradients
# ---------------------------------------------------------------------------
def make_cores(cfg: TTConfig, seed: int = 0, mixed_magnitude: bool = False
               ) -> List[Tuple[np.ndarray, np.ndarray, np.ndarray]]:
    """Per table (C1[m1][n1][R], C2[m2][R][n2][R], C3[m3][R][n3]) float32; a dense (hybrid)
    table is (W[M][N] ~ U(-1/sqrt(N), 1/sqrt(N)), empty, empty).

    DESIGN.md R21: C1 ~ U(-1,1), C2, C3 ~ U(-1/sqrt(R), 1/sqrt(R)).
    mixed_magnitude scales a seeded 10% of C2 slices by 1e3 (exercises the
    relative-error metric)."""
    n1, n2, n3 = cfg.col_factors
    R = cfg.rank
    a = 1.0 / np.sqrt(R)
    out = []
    for t, (m1, m2, m3) in enumerate(cfg.row_factors):
        g = rng("cores", cfg.name, seed, t)
        if cfg.is_dense(t):
            N = n1 * n2 * n3
            w = g.uniform(-1.0, 1.0, size=(cfg.table_rows[t], N)) / np.sqrt(N)
            out.append((w.astype(np.float32), np.zeros((0, R, n2, R), np.float32),
                        np.zeros((0, R, n3), np.float32)))
            continue
        c1 = g.uniform(-1.0, 1.0, size=(m1, n1, R)).astype(np.float32)
        c2 = g.uniform(-a, a, size=(m2, R, n2, R)).astype(np.float32)
        c3 = g.uniform(-a, a, size=(m3, R, n3)).astype(np.float32)
        if mixed_magnitude:
            sel = g.random(m2) < 0.1
            c2[sel] *= np.float32(1e3)
        out.append((c1, c2, c3))
    return out


def make_grad_out(cfg: TTConfig, batch: int, step: int = 0, seed: int = 0) -> np.ndarray:
    """Upstream gradient dL/d out, float32 [B][T][N], U(-1, 1)."""
    g = rng("grad_out", cfg.name, seed, step, batch)
    return g.uniform(-1.0, 1.0, size=(batch, cfg.num_tables, cfg.dim)).astype(np.float32)


def core_bytes(cfg: TTConfig) -> int:
    n1, n2, n3 = cfg.col_factors
    R = cfg.rank
    tot = 0
    for t, (m1, m2, m3) in enumerate(cfg.row_factors):
        if cfg.is_dense(t):
            tot += cfg.table_rows[t] * n1 * n2 * n3
        else:
            tot += m1 * n1 * R + m2 * R * n2 * R + m3 * R * n3
    return 4 * tot


def small_config(table_rows: Sequence[int], row_factors: Sequence[Tuple[int, int, int]],
                 col_factors: Tuple[int, int, int], rank: int, batch: int, pooling: int = 1,
                 zipf_s: Optional[float] = None, name: str = "small",
                 id_map: str = "identity") -> TTConfig:
    """Ad-hoc config for tests (explicit factors)."""
    return _mk(name, table_rows, col_factors, rank, batch, pooling, zipf_s,
               factors=row_factors, id_map=id_map)


def make_host_batch(table_rows: Sequence[int], batch: int, pooling: int, zipf_s: Optional[float],
                    step: int = 0, seed: int = 0, name: str = "host") -> Tuple[np.ndarray, np.ndarray]:
    """Ids of the host-memory tables of the pipeline (f4; P:417 keeps all but the largest table
    in host memory): (indices int64, offsets int64 [T*B+1]), table-major, fixed bag length,
    Zipf ids so consecutive batches share hot rows (the RAW hazard of P:296)."""
    T = len(table_rows)
    offsets = np.arange(T * batch + 1, dtype=np.int64) * pooling
    parts = [zipf_ids(rng("host_ids", name, seed, step, t), int(table_rows[t]), zipf_s, batch * pooling)
             for t in range(T)]
    return (np.concatenate(parts) if parts else np.zeros(0, dtype=np.int64)), offsets


def make_host_weight(table_rows: Sequence[int], dim: int, seed: int = 0) -> np.ndarray:
    """Initial host-table parameters, float32 [sum rows][dim], U(-0.05, 0.05)."""
    return rng("host_w", seed, dim, *[int(r) for r in table_rows]).uniform(
        -0.05, 0.05, size=(int(sum(table_rows)), dim)).astype(np.float32)


def make_host_grad_out(num_tables: int, batch: int, dim: int, step: int = 0, seed: int = 0) -> np.ndarray:
    """Upstream gradient of the host-table outputs, float32 [B][T][dim], U(-1, 1)."""
    return rng("host_go", seed, step, batch, num_tables, dim).uniform(
        -1.0, 1.0, size=(batch, num_tables, dim)).astype(np.float32)
