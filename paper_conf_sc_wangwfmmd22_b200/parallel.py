"""Data-parallel plumbing for the TT-EmbeddingBag.

TT cores are replicated on every rank; rank g owns samples [g*B/G, (g+1)*B/G) of every
table.  After `ttemb_backward` (non-fused) the dense core-gradient buffer is summed across
ranks with one all-reduce ("the only communication is the gradient all-reduce") and
every replica applies the same update, so replicas stay bitwise identical.
"""
from __future__ import annotations

from typing import Optional, Tuple

import numpy as np
import torch
import torch.distributed as dist


def shard_bags(indices: np.ndarray, offsets: np.ndarray, num_tables: int, batch: int, rank: int,
               world: int) -> Tuple[np.ndarray, np.ndarray, int]:
    """Host-side batch partition: this rank's (indices, offsets rebased to 0, local batch)
    from a global table-major batch (offsets [T*B+1])."""
    if world < 1 or not 0 <= rank < world:
        raise ValueError("bad rank / world")
    if batch % world:
        raise ValueError("global batch must be divisible by the world size")
    bl = batch // world
    b0 = rank * bl
    offsets = np.asarray(offsets, dtype=np.int64)
    parts, lens = [], []
    for t in range(num_tables):
        lo, hi = t * batch + b0, t * batch + b0 + bl
        parts.append(np.asarray(indices[offsets[lo]:offsets[hi]]))
        lens.append(np.diff(offsets[lo:hi + 1]))
    off = np.zeros(num_tables * bl + 1, dtype=np.int64)
    if lens:
        np.cumsum(np.concatenate(lens), out=off[1:])
    idx = np.concatenate(parts) if parts else np.zeros(0, dtype=np.int64)
    return idx.astype(np.asarray(indices).dtype, copy=False), off, bl


def allreduce_grads(grads: torch.Tensor, group: Optional[dist.ProcessGroup] = None) -> None:
    """SUM all-reduce of the dense core-gradient buffer, in place (NCCL on GPUs)."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(grads, op=dist.ReduceOp.SUM, group=group)


def dp_step(emb, indices: torch.Tensor, offsets: torch.Tensor, batch: int, grad_out_fn, lr: float,
            group: Optional[dist.ProcessGroup] = None, out: Optional[torch.Tensor] = None):
    """One data-parallel step on this rank: forward, backward (dense grads), all-reduce,
    update.  `grad_out_fn(out)` returns dL/d out (e.g. the rest of the model's backward).
    The embedding must have been created with fused_update=False."""
    if emb.fused:
        raise ValueError("data-parallel steps need fused_update=False (update after all-reduce)")
    out = emb.forward(indices, offsets, batch, out=out)
    emb.backward(grad_out_fn(out))
    allreduce_grads(emb.grads, group)
    emb.update(lr)
    return out
