"""Host-memory tier of EL-Rec's pipeline training system (PAPER §V).

Embedding tables that do not fit in HBM are kept in (pinned) host memory.  A CPU parameter
server pre-fetches the rows of the next batches into a Pre-fetch Queue and applies the gradients
the GPU worker pushes into a Gradient Queue (Fig. 9).  With a queue length L > 1 the two
overlap, and a batch may be pre-fetched before the updates of the previous batches reached host
memory: the read-after-write conflict of P:294-296.  The GPU embedding cache (index table + life
cycles) keeps every row the last batches updated and overwrites the stale copies, so
pipelined training computes exactly what sequential training (L = 1) computes.

Schedule (reading R31): the server pre-fetches batch k only after it has applied the
gradients of batch k - L (L = 1: strictly sequential, "the GPU-side training workers can only
wait for the CPU side finishing parameter update").  A row updated by batch j can then be
stale only in batches j+1 .. j+L-1; the worker pushes it into the cache with LC = L and every
trained batch is one gradient-queue pull (LC -= 1), so it is still cached when those batches
synchronise.  Cache capacity L * max_unique rows is therefore always enough.

Every step of the data path runs in libttemb.so: the device kernels (ttemb_ht_sync / pool /
grad / tick / update_push) and the native multi-threaded host gather / SGD of the server
(ttemb_ht_host_gather / ttemb_ht_host_sgd).  Python keeps the queues and issues the copies.
"""
from __future__ import annotations

import ctypes as C
import queue
import threading
import time
from dataclasses import dataclass
from typing import Callable, List, Optional, Sequence, Tuple

import numpy as np
import torch

from . import _lib as L
from ._lib import check


@dataclass
class HostBatch:
    """A batch's host-tier part as the server prepares it ("indices and parameters")."""
    ids: np.ndarray        # int64 [U]   distinct global host rows, ascending
    ridx: np.ndarray       # int32 [nnz] block row of each position
    offsets: np.ndarray    # int64 [T*B+1] table-major bags
    occ_ptr: np.ndarray    # int64 [U+1] positions of row u: occ_bag[occ_ptr[u]:occ_ptr[u+1]]
    occ_bag: np.ndarray    # int32 [nnz] bag (t*B+b) of each occurrence, in position order


def prepare_batch(indices: np.ndarray, offsets: np.ndarray, table_base: np.ndarray, batch: int) -> HostBatch:
    """Server-side index preparation: global row ids, the unique block, occurrence lists."""
    T = len(table_base) - 1
    offsets = np.asarray(offsets, dtype=np.int64)
    indices = np.asarray(indices, dtype=np.int64)
    nnz = int(offsets[-1])
    lengths = np.diff(offsets)
    bag = np.repeat(np.arange(T * batch, dtype=np.int64), lengths)
    tab = bag // batch
    rows_t = np.diff(table_base)
    if nnz and (np.any(indices < 0) or np.any(indices >= rows_t[tab])):
        raise ValueError("host-tier id outside its table")
    gid = indices + table_base[:-1][tab]
    # one sort of (row, position) keys gives the unique ids, the inverse and the occurrence lists
    # in position order (a packed key sorts ~10x faster than numpy's stable argsort)
    if int(table_base[-1]) * max(nnz, 1) < 2 ** 62:
        key = np.sort(gid * max(nnz, 1) + np.arange(nnz, dtype=np.int64))
        sg, order = np.divmod(key, max(nnz, 1))
    else:
        order = np.argsort(gid, kind="stable")
        sg = gid[order]
    first = np.empty(nnz, dtype=bool)
    if nnz:
        first[0] = True
        np.not_equal(sg[1:], sg[:-1], out=first[1:])
    starts = np.flatnonzero(first)
    inv = np.empty(nnz, dtype=np.int32)
    inv[order] = np.cumsum(first) - 1
    occ_ptr = np.append(starts, nnz).astype(np.int64)
    return HostBatch(sg[starts].astype(np.int64), inv, offsets, occ_ptr, bag[order].astype(np.int32))


class _Slot:
    """Pinned host staging + device buffers of one in-flight batch."""

    def __init__(self, max_u: int, max_nnz: int, nbags: int, dim: int, dev: torch.device):
        pin = dict(pin_memory=True)
        self.h_rows = torch.empty(max_u, dim, dtype=torch.float32, **pin)
        self.h_ids = torch.empty(max_u, dtype=torch.int64, **pin)
        self.h_ridx = torch.empty(max_nnz, dtype=torch.int32, **pin)
        self.h_off = torch.empty(nbags + 1, dtype=torch.int64, **pin)
        self.h_optr = torch.empty(max_u + 1, dtype=torch.int64, **pin)
        self.h_obag = torch.empty(max_nnz, dtype=torch.int32, **pin)
        self.h_grad = torch.empty(max_u, dim, dtype=torch.float32, **pin)
        self.rows = torch.empty(max_u, dim, dtype=torch.float32, device=dev)
        self.ids = torch.empty(max_u, dtype=torch.int64, device=dev)
        self.ridx = torch.empty(max_nnz, dtype=torch.int32, device=dev)
        self.off = torch.empty(nbags + 1, dtype=torch.int64, device=dev)
        self.optr = torch.empty(max_u + 1, dtype=torch.int64, device=dev)
        self.obag = torch.empty(max_nnz, dtype=torch.int32, device=dev)
        self.g = torch.empty(max_u, dim, dtype=torch.float32, device=dev)
        self.U = 0
        self.nnz = 0
        self.ready = torch.cuda.Event()     # H2D of the pre-fetch done
        self.pushed = torch.cuda.Event()    # D2H of the gradients done


def _ptr(t: torch.Tensor) -> int:
    return t.data_ptr()


class HostTierEmbedding:
    """Sum-pooled embedding bags over host-memory tables, trained by SGD through the pipeline.

    host_rows   rows of each host table (all share `dim`); the parameters are
                `self.weight` (pinned float32 [sum rows][dim], table t at rows
                table_base[t] .. table_base[t+1]).
    queue_len   L: pre-fetch depth = gradient-queue length = cache life cycle.
    use_cache   False disables the synchronisation (the RAW-conflict ablation of P:296).
    threaded    True: the server is a thread running ahead on its own; False: the same server
                steps run inline at the earliest point the schedule allows (deterministic,
                maximally stale pre-fetches; used by the tests).
    """

    def __init__(self, host_rows: Sequence[int], dim: int, batch: int, max_nnz: int, queue_len: int,
                 lr: float, device: int = 0, use_cache: bool = True, threaded: bool = True,
                 server_threads: int = 0, weight: Optional[np.ndarray] = None):
        L.load()
        if queue_len < 1:
            raise ValueError("queue_len >= 1")
        self.T = len(host_rows)
        self.dim, self.B, self.max_nnz, self.L, self.lr = int(dim), int(batch), int(max_nnz), int(queue_len), float(lr)
        self.table_base = np.zeros(self.T + 1, dtype=np.int64)
        np.cumsum(np.asarray(host_rows, dtype=np.int64), out=self.table_base[1:])
        self.n_rows = int(self.table_base[-1])
        self.dev = torch.device("cuda", device)
        self.use_cache, self.threaded, self.server_threads = bool(use_cache), bool(threaded), int(server_threads)
        self.weight = torch.empty(self.n_rows, self.dim, dtype=torch.float32, pin_memory=True)
        if weight is not None:
            self.weight.numpy()[:] = np.asarray(weight, dtype=np.float32).reshape(self.n_rows, self.dim)
        else:
            self.weight.zero_()
        max_u = self.max_nnz
        self.capacity = max(1, self.L * max_u)
        i32, i64, f32 = torch.int32, torch.int64, torch.float32
        self.c_index = torch.empty(max(self.n_rows, 1), dtype=i32, device=self.dev)
        self.c_rows = torch.empty(self.capacity, self.dim, dtype=f32, device=self.dev)
        self.c_lc = torch.empty(self.capacity, dtype=i32, device=self.dev)
        self.c_owner = torch.zeros(self.capacity, dtype=i64, device=self.dev)
        self.c_free = torch.empty(self.capacity, dtype=i32, device=self.dev)
        self.c_top = torch.empty(2, dtype=i32, device=self.dev)
        self.cache = L.ttemb_ht_cache(_ptr(self.c_index), _ptr(self.c_rows), _ptr(self.c_lc), _ptr(self.c_owner),
                                      _ptr(self.c_free), _ptr(self.c_top), self.n_rows, self.capacity, self.dim)
        self._cp = C.byref(self.cache)
        self.h2d_stream = torch.cuda.Stream(device=self.dev)     # server: pre-fetch copies
        self.d2h_stream = torch.cuda.Stream(device=self.dev)     # worker: gradient-queue copies
        self.slots = [_Slot(max_u, self.max_nnz, self.T * self.B, self.dim, self.dev) for _ in range(self.L + 1)]
        check(L._lib.ttemb_ht_cache_init(self._cp, torch.cuda.current_stream(self.dev).cuda_stream), "ht_cache_init")
        self._reset_queues()

    # -- queues / server ---------------------------------------------------------------------
    def _reset_queues(self):
        self.prefetch_q: "queue.Queue" = queue.Queue()
        self.grad_q: "queue.Queue" = queue.Queue()
        self.applied = 0
        self.prefetched = 0
        self.steps = 0
        self.source = None
        self._server = None
        self._error: Optional[BaseException] = None
        # host seconds: server pre-fetch (index prep + gather + copy issue), server apply (wait for
        # the gradient copy + SGD), worker blocked on the pre-fetch queue
        self.times = {"prefetch": 0.0, "apply": 0.0, "worker_wait": 0.0}

    def start(self, source: Callable[[int], Tuple[np.ndarray, np.ndarray]], steps: int) -> None:
        """source(k) -> (indices int64, offsets int64 [T*B+1]) of the host tables for batch k."""
        torch.cuda.synchronize(self.dev)
        self._reset_queues()
        self.source, self.steps = source, int(steps)
        if self.threaded:
            self._applied_cv = threading.Condition()
            self._server = [threading.Thread(target=self._serve_prefetch, daemon=True),
                            threading.Thread(target=self._serve_apply, daemon=True)]
            for th in self._server:
                th.start()
        else:
            for k in range(min(self.L, self.steps)):
                self._prefetch(k)

    # The server runs as two threads: the pre-fetcher waits only for the one ordering rule (batch
    # k - L applied before batch k is gathered), the applier pulls gradients as they arrive.  A
    # gather may then read a row while the applier updates it -- only rows of batches after k - L,
    # which the cache holds and k_ht_sync overwrites, so a torn or stale read there is harmless.
    def _serve_prefetch(self):
        try:
            torch.cuda.set_device(self.dev)
            for k in range(self.steps):
                with self._applied_cv:
                    self._applied_cv.wait_for(lambda: self.applied >= k - self.L + 1 or self._error is not None)
                if self._error is not None:
                    return
                self._prefetch(k)
        except BaseException as e:                        # surfaced by forward / finish
            self._error = e
            self.prefetch_q.put(None)

    def _serve_apply(self):
        try:
            torch.cuda.set_device(self.dev)
            while self.applied < self.steps:
                self._apply_one()
                with self._applied_cv:
                    self._applied_cv.notify_all()
        except BaseException as e:
            self._error = e
            self.prefetch_q.put(None)
            with self._applied_cv:
                self._applied_cv.notify_all()

    def _prefetch(self, k: int) -> None:
        """Server: gather batch k's rows from host memory into its slot and copy them to HBM."""
        t0 = time.perf_counter()
        idx, off = self.source(k)
        hb = prepare_batch(idx, off, self.table_base, self.B)
        U, nnz = len(hb.ids), int(hb.offsets[-1])
        if nnz > self.max_nnz:
            raise ValueError("batch exceeds max_nnz")
        s = self.slots[k % len(self.slots)]
        s.U, s.nnz = U, nnz
        s.h_ids.numpy()[:U] = hb.ids
        s.h_ridx.numpy()[:nnz] = hb.ridx
        s.h_off.numpy()[:] = hb.offsets
        s.h_optr.numpy()[:U + 1] = hb.occ_ptr
        s.h_obag.numpy()[:nnz] = hb.occ_bag
        check(L._lib.ttemb_ht_host_gather(_ptr(self.weight), self.n_rows, self.dim, _ptr(s.h_ids), U,
                                          _ptr(s.h_rows), self.server_threads), "ht_host_gather")
        with torch.cuda.stream(self.h2d_stream):
            s.rows[:U].copy_(s.h_rows[:U], non_blocking=True)
            s.ids[:U].copy_(s.h_ids[:U], non_blocking=True)
            s.ridx[:nnz].copy_(s.h_ridx[:nnz], non_blocking=True)
            s.off.copy_(s.h_off, non_blocking=True)
            s.optr[:U + 1].copy_(s.h_optr[:U + 1], non_blocking=True)
            s.obag[:nnz].copy_(s.h_obag[:nnz], non_blocking=True)
            s.ready.record(self.h2d_stream)
        self.prefetched = k + 1
        self.times["prefetch"] += time.perf_counter() - t0
        self.prefetch_q.put(k)

    def _apply_one(self) -> None:
        """Server: pull one batch from the gradient queue and apply it to host memory."""
        k = self.grad_q.get()
        t0 = time.perf_counter()
        s = self.slots[k % len(self.slots)]
        s.pushed.synchronize()
        check(L._lib.ttemb_ht_host_sgd(_ptr(self.weight), self.n_rows, self.dim, _ptr(s.h_ids), s.U,
                                       _ptr(s.h_grad), self.lr, self.server_threads), "ht_host_sgd")
        self.applied = k + 1
        self.times["apply"] += time.perf_counter() - t0

    # -- worker ------------------------------------------------------------------------------
    def forward(self, k: int, out: Optional[torch.Tensor] = None) -> torch.Tensor:
        """Pop batch k from the pre-fetch queue, synchronise it with the cache (Step 1)
        and pool it: out [B][T][dim] float32 on the current stream."""
        t0 = time.perf_counter()
        got = self.prefetch_q.get()
        self.times["worker_wait"] += time.perf_counter() - t0
        if got is None or self._error is not None:
            raise RuntimeError("host-tier server failed") from self._error
        assert got == k, (got, k)
        s = self.slots[k % len(self.slots)]
        st = torch.cuda.current_stream(self.dev)
        st.wait_event(s.ready)
        sp = st.cuda_stream
        if self.use_cache:
            check(L._lib.ttemb_ht_sync(self._cp, _ptr(s.ids), s.U, _ptr(s.rows), sp), "ht_sync")
        if out is None:
            out = torch.empty(self.B, self.T, self.dim, dtype=torch.float32, device=self.dev)
        check(L._lib.ttemb_ht_pool(_ptr(s.rows), _ptr(s.ridx), _ptr(s.off), self.T, self.B, self.dim,
                                   _ptr(out), sp), "ht_pool")
        self._cur = k
        return out

    def backward(self, grad_out: torch.Tensor) -> None:
        """Row gradients, SGD on the block, cache push (LC = L) after one LC tick, and the
        gradients into the Gradient Queue (Step 3)."""
        k = self._cur
        s = self.slots[k % len(self.slots)]
        assert grad_out.is_contiguous() and grad_out.shape == (self.B, self.T, self.dim)
        st = torch.cuda.current_stream(self.dev)
        sp = st.cuda_stream
        check(L._lib.ttemb_ht_grad(_ptr(grad_out), _ptr(s.optr), _ptr(s.obag), s.U, self.T, self.B, self.dim,
                                   _ptr(s.g), sp), "ht_grad")
        if self.use_cache:
            check(L._lib.ttemb_ht_tick(self._cp, sp), "ht_tick")
        check(L._lib.ttemb_ht_update_push(self._cp, _ptr(s.rows), _ptr(s.g), _ptr(s.ids), s.U, self.lr,
                                          self.L if self.use_cache else 0, sp), "ht_update_push")
        self.d2h_stream.wait_stream(st)
        with torch.cuda.stream(self.d2h_stream):
            s.h_grad[:s.U].copy_(s.g[:s.U], non_blocking=True)
            s.pushed.record(self.d2h_stream)
        self.grad_q.put(k)
        if not self.threaded:                 # inline server: apply k, then pre-fetch k + L
            self._apply_one()
            if k + self.L < self.steps:
                self._prefetch(k + self.L)

    def finish(self) -> None:
        """Drain: the server applies every pushed gradient; host memory is then current."""
        if self._server is not None:
            for th in self._server:
                th.join()
            self._server = None
        if self._error is not None:
            raise RuntimeError("host-tier server failed") from self._error
        while self.applied < self.steps and not self.grad_q.empty():
            self._apply_one()
        torch.cuda.synchronize(self.dev)

    def cache_stats(self) -> Tuple[int, int]:
        """(live cache entries, overflow flag)."""
        live, ovf = C.c_int32(), C.c_int32()
        check(L._lib.ttemb_ht_cache_stats(self._cp, C.byref(live), C.byref(ovf),
                                          torch.cuda.current_stream(self.dev).cuda_stream), "ht_cache_stats")
        return live.value, ovf.value
