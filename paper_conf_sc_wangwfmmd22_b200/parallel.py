"""Data-parallel plumbing for the TT-EmbeddingBag.

TT cores are replicated on every rank; rank g owns samples [g*B/G, (g+1)*B/G) of every
table (the host-side partition is `synth.workload.shard_batch`, part of the input recipe).
After an unfused `ttemb_backward` the dense core-gradient buffer is summed across ranks ("the
only communication is the gradient all-reduce") and every replica applies the same
update, so replicas stay bitwise identical (the SUM is the same reduction on every rank).

`GradSync` does that exchange in one of two ways:

* ``allreduce``: the gradient buffer is all-reduced bucket by bucket on a communication
  stream.  The backward records one CUDA event per bucket as soon as the bucket is final
  (`ttemb_set_bucket_events`: dense tables after the aggregation, every C3 core after the row
  stage, C1 + C2 at the end), so the early buckets travel while the prefix-backward kernel
  still runs; then every rank applies the full update (`ttemb_update`).
* ``rs_ag``: reduce-scatter of the (padded) buffer, each rank updates only its 1/G shard
  (`ttemb_update_range`; the Adagrad state of the other shards is never touched), then an
  all-gather of the updated cores.  Same wire bytes as the all-reduce; the update traffic and the
  live optimizer state per rank shrink by G.

Everything is enqueued on CUDA streams with events (no host synchronisation), so a data-parallel
step can be captured in a CUDA graph with NCCL.  With the gloo backend (CPU tests, ranks sharing
one GPU) the collectives run synchronously on the current stream, and gloo's missing
reduce-scatter is emulated by an all-reduce (identical result).
"""
from __future__ import annotations

from typing import List, Optional, Tuple

import torch
import torch.distributed as dist


def allreduce_grads(grads: torch.Tensor, group: Optional[dist.ProcessGroup] = None) -> None:
    """SUM all-reduce of the dense core-gradient buffer, in place (NCCL on GPUs)."""
    if dist.is_available() and dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(grads, op=dist.ReduceOp.SUM, group=group)


def shard_range(n: int, world: int, rank: int) -> Tuple[int, int]:
    """Equal shards of a flat buffer of n floats (n divisible by world): (begin, count)."""
    if n % world:
        raise ValueError("flat buffer length must be divisible by the world size")
    c = n // world
    return rank * c, c


class GradSync:
    """Gradient exchange + update of one replicated TTEmbeddingBag (unfused) per step."""

    def __init__(self, emb, mode: str = "allreduce", group: Optional[dist.ProcessGroup] = None,
                 comm_stream: Optional[torch.cuda.Stream] = None):
        if emb.fused:
            raise ValueError("data-parallel steps need fused_update=False (update after the exchange)")
        if mode not in ("allreduce", "rs_ag"):
            raise ValueError(mode)
        self.emb, self.mode, self.group = emb, mode, group
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.backend = dist.get_backend(group) if dist.is_initialized() else "none"
        self.async_comm = self.backend == "nccl" and emb.grads.is_cuda
        self.buckets: List[Tuple[int, int]] = [b for b in emb.grad_buckets() if b[1] > 0] \
            if mode == "allreduce" else []
        self.comm = comm_stream if comm_stream is not None else (
            torch.cuda.Stream(device=emb.device) if self.async_comm else None)
        if mode == "allreduce" and self.async_comm:
            ev = [torch.cuda.Event() for _ in range(3)]
            emb.set_bucket_events(ev)
            nb = emb.grad_buckets()
            self._events = [ev[i] for i, b in enumerate(nb) if b[1] > 0]
        else:
            self._events = []

    # -- the step -------------------------------------------------------------------------
    def exchange_and_update(self, lr: float) -> None:
        """Call right after `emb.backward(...)` on the compute stream."""
        if self.world == 1:
            self.emb.update(lr)
            return
        if self.mode == "allreduce":
            self._allreduce()
            self.emb.update(lr)
        else:
            self._rs_update_ag(lr)

    def _allreduce(self) -> None:
        g = self.emb.grads
        if not self.async_comm:
            dist.all_reduce(g, op=dist.ReduceOp.SUM, group=self.group)
            return
        cur = torch.cuda.current_stream(g.device)
        with torch.cuda.stream(self.comm):
            for (b, n), ev in zip(self.buckets, self._events):
                self.comm.wait_event(ev)          # bucket final on the compute stream
                dist.all_reduce(g[b:b + n], op=dist.ReduceOp.SUM, group=self.group)
        cur.wait_stream(self.comm)

    def _rs_update_ag(self, lr: float) -> None:
        emb = self.emb
        g, c = emb.grads, emb.cores
        b, n = shard_range(g.numel(), self.world, self.rank)
        if self.backend == "nccl":
            out = g[b:b + n]
            dist.reduce_scatter_tensor(out, g, op=dist.ReduceOp.SUM, group=self.group)
        else:                                      # gloo: no reduce-scatter; same SUM per shard
            dist.all_reduce(g, op=dist.ReduceOp.SUM, group=self.group)
        emb.update_range(lr, b, n)
        if self.backend == "nccl":
            dist.all_gather_into_tensor(c, c[b:b + n].clone(), group=self.group)
        else:                                      # gloo all-gathers host tensors only
            mine = c[b:b + n].cpu()
            parts = [torch.empty_like(mine) for _ in range(self.world)]
            dist.all_gather(parts, mine, group=self.group)
            c.copy_(torch.cat(parts).to(c.device))
