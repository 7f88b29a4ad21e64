"""Data-parallel plumbing for the TT-EmbeddingBag.

TT cores are replicated on every rank; rank g owns samples [g*B/G, (g+1)*B/G) of every
table (the host-side partition is `synth.workload.shard_batch`, part of the input recipe).  After `ttemb_backward` (non-fused) the dense core-gradient buffer is summed across
ranks with one all-reduce ("the only communication is the gradient all-reduce") and
every replica applies the same update, so replicas stay bitwise identical.
"""
from __future__ import annotations

from typing import Optional

import torch
import torch.distributed as dist


def allreduce_grads(grads: torch.Tensor, group: Optional[dist.ProcessGroup] = None) -> None:
    """SUM all-reduce of the dense core-gradient buffer, in place (NCCL on GPUs)."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(grads, op=dist.ReduceOp.SUM, group=group)
