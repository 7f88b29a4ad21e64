"""Oracle of the host-memory tier (PAPER §V).

TEST INFRASTRUCTURE ONLY: imported by tests/ (and scripts that check results), never by the
product package; it imports nothing from it.

What the pipeline must compute: sum-pooled embedding bags over plain tables (Eq. 4 with plain
rows), trained by SGD, batch after batch -- i.e. SEQUENTIAL training; the embedding cache exists
so that pipelined pre-fetching changes nothing ("after embedding synchronization, all
embeddings are up to date").  `train_stale` is the same pipeline WITHOUT the cache: batch k reads
host memory as it stood when it was pre-fetched, after the gradients of batches <= k - L had been
applied (the schedule of DESIGN.md R31), which is the read-after-write conflict of P:294-296.

Precision: float32 in the product's order, so the comparison can be bit-exact -- every pooled
sum and every row gradient is accumulated from 0 in position order, one float32 rounding per
addition; SGD is w - rn(lr * g) (two roundings, no fused multiply-add).  Written with plain
loops over bags / positions (small cases only).

Pins (tests/test_hosttier.py): forward, gradients and SGD against torch.nn.EmbeddingBag
(mode="sum") + autograd + torch.optim.SGD in float64; stale training with L = 1 equals sequential
training; stale training differs from it exactly when consecutive batches share rows.
"""
from __future__ import annotations

from typing import Callable, List, Sequence, Tuple

import numpy as np


def _bags(offsets: np.ndarray, T: int, B: int):
    for t in range(T):
        for b in range(B):
            yield t, b, int(offsets[t * B + b]), int(offsets[t * B + b + 1])


def forward(W: np.ndarray, table_base: Sequence[int], indices: np.ndarray, offsets: np.ndarray,
            B: int) -> np.ndarray:
    """out[b][t] = sum over the bag's positions j (in order) of W[table_base[t] + indices[j]]."""
    T = len(table_base) - 1
    N = W.shape[1]
    out = np.zeros((B, T, N), dtype=np.float32)
    for t, b, j0, j1 in _bags(offsets, T, B):
        acc = np.zeros(N, dtype=np.float32)
        for j in range(j0, j1):
            acc = acc + W[table_base[t] + indices[j]]          # float32 + float32, rounded
        out[b, t] = acc
    return out


def row_grads(grad_out: np.ndarray, table_base: Sequence[int], indices: np.ndarray, offsets: np.ndarray,
              B: int) -> Tuple[np.ndarray, np.ndarray]:
    """dL/dW[r] for L = sum(out * grad_out): (rows ascending, g[rows]), each g summed over the
    row's positions in position order."""
    T = len(table_base) - 1
    N = grad_out.shape[2]
    acc = {}
    for t, b, j0, j1 in _bags(offsets, T, B):
        for j in range(j0, j1):
            r = int(table_base[t] + indices[j])
            acc[r] = (acc[r] if r in acc else np.zeros(N, dtype=np.float32)) + grad_out[b, t]
    rows = np.array(sorted(acc), dtype=np.int64)
    g = np.stack([acc[r] for r in rows]) if len(rows) else np.zeros((0, N), dtype=np.float32)
    return rows, g.astype(np.float32)


def squared_loss_grad(targets: List[np.ndarray]) -> Callable[[int, np.ndarray], np.ndarray]:
    """grad_fn of L_k = 1/2 |out_k - y_k|^2: dL/dout = out - y (one float32 subtraction)."""
    return lambda k, out: (out - targets[k]).astype(np.float32)


def sgd(W: np.ndarray, rows: np.ndarray, g: np.ndarray, lr: float) -> None:
    """W[r] <- W[r] - rn(lr * g_r), in place (plain SGD)."""
    W[rows] = W[rows] - np.float32(lr) * g


def train_sequential(W0: np.ndarray, table_base, batches: List[Tuple[np.ndarray, np.ndarray]],
                     grad_fn: Callable[[int, np.ndarray], np.ndarray], B: int, lr: float):
    """Queue length 1: returns (final W, [out_k]).  grad_fn(k, out_k) -> dL/dout_k (the
    model above the embedding layer; with a loss that is linear in out the gradients would not
    depend on the parameters and stale reads could not change the weights)."""
    W = np.array(W0, dtype=np.float32, copy=True)
    outs = []
    for k, (idx, off) in enumerate(batches):
        outs.append(forward(W, table_base, idx, off, B))
        rows, g = row_grads(grad_fn(k, outs[-1]), table_base, idx, off, B)
        sgd(W, rows, g, lr)
    return W, outs


def train_stale(W0: np.ndarray, table_base, batches, grad_fn, B: int, lr: float, L: int):
    """Pipeline of queue length L without the embedding cache: batch k is trained on the host
    state after batches 0 .. k-L were applied; its gradients are applied to the current state."""
    W = np.array(W0, dtype=np.float32, copy=True)
    snaps = {}
    outs = []
    for k, (idx, off) in enumerate(batches):
        if k - L + 1 <= 0:
            snaps[k] = np.array(W0, dtype=np.float32, copy=True)
        view = snaps.pop(k)
        outs.append(forward(view, table_base, idx, off, B))
        rows, g = row_grads(grad_fn(k, outs[-1]), table_base, idx, off, B)
        sgd(W, rows, g, lr)
        if k + L < len(batches):
            snaps[k + L] = W.copy()                     # pre-fetch of batch k + L, after applying k
    return W, outs
