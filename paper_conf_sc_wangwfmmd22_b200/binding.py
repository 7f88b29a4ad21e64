"""Thin Python binding over libttemb.so (include/ttemb.h).

The module-level functions carry the C names (ttemb_create, ttemb_forward, ...)
and only marshal arguments.  `TTEmbeddingBag` is a convenience owner of the
caller-side buffers: PyTorch provides device memory and streams, nothing else
(every step of the path runs in the library's kernels).
"""
from __future__ import annotations

import ctypes as C
from typing import Dict, List, Optional, Sequence, Tuple

import numpy as np
import torch

from . import _lib as L
from ._lib import TTEmbError, check

STAGES: List[str] = []


def _stream_ptr(stream: Optional[torch.cuda.Stream]) -> int:
    s = stream if stream is not None else torch.cuda.current_stream()
    return int(s.cuda_stream)


def make_config(table_rows: Sequence[int], row_factors: Sequence[Tuple[int, int, int]],
                col_factors: Tuple[int, int, int], rank: int, max_batch: int, max_nnz: int,
                optimizer: str = "sgd", adagrad_eps: float = 1e-10, fused_update: bool = False,
                index_bits: int = 64, num_cores: int = 3, fp32_cores: bool = False,
                prefix_reuse: bool = True, aggregation: bool = True, mode: str = "sum",
                dense: Sequence[bool] = ()):
    """Returns (ttemb_config, keep-alive table array).  mode = "sum" | "mean" (nn.EmbeddingBag);
    dense[t] keeps table t uncompressed (hybrid placement).  prefix_reuse / aggregation = False set the
    ablation flags TTEMB_NO_PREFIX_REUSE / TTEMB_NO_AGGREGATION."""
    T = len(table_rows)
    tabs = (L.ttemb_table * max(T, 1))()
    for t in range(T):
        tabs[t].num_rows = int(table_rows[t])
        tabs[t].dense = 1 if (len(dense) and dense[t]) else 0
        for k in range(3):
            tabs[t].row_factors[k] = int(row_factors[t][k])
    cfg = L.ttemb_config()
    cfg.num_tables = T
    cfg.tables = C.cast(tabs, C.POINTER(L.ttemb_table))
    cfg.num_cores = int(num_cores)
    cfg.dim = int(np.prod(col_factors))
    for k in range(3):
        cfg.col_factors[k] = int(col_factors[k])
    cfg.rank = int(rank)
    cfg.index_bits = int(index_bits)
    cfg.max_batch = int(max_batch)
    cfg.max_nnz = int(max_nnz)
    cfg.optimizer = {"sgd": L.TTEMB_SGD, "adagrad": L.TTEMB_ADAGRAD}[optimizer]
    cfg.adagrad_eps = float(adagrad_eps)
    cfg.flags = ((L.TTEMB_FUSED_UPDATE if fused_update else 0) | (L.TTEMB_FP32_CORES if fp32_cores else 0)
                 | (0 if prefix_reuse else L.TTEMB_NO_PREFIX_REUSE)
                 | (0 if aggregation else L.TTEMB_NO_AGGREGATION)
                 | {"sum": 0, "mean": L.TTEMB_MEAN_POOLING}[mode])
    return cfg, tabs


# ---------------------------------------------------------------------------
# Same-name wrappers of the C ABI
# ---------------------------------------------------------------------------
def ttemb_query_sizes(cfg) -> Tuple[int, int, int, int]:
    v = [C.c_size_t() for _ in range(4)]
    check(L.load().ttemb_query_sizes(C.byref(cfg), *[C.byref(x) for x in v]), "ttemb_query_sizes")
    return tuple(int(x.value) for x in v)


def ttemb_create(cfg, device: int, cores: int, state: int, grads: int, workspace: int) -> int:
    h = C.c_void_p()
    check(L.load().ttemb_create(C.byref(cfg), int(device), cores, state or None, grads, workspace,
                                C.byref(h)), "ttemb_create")
    return h.value


def ttemb_destroy(h: int) -> None:
    check(L.load().ttemb_destroy(h), "ttemb_destroy")


def ttemb_core_layout(h: int, table: int, core: int) -> Tuple[int, Tuple[int, int, int, int]]:
    off = C.c_int64()
    shape = (C.c_int32 * 4)()
    check(L.load().ttemb_core_layout(h, table, core, C.byref(off), shape), "ttemb_core_layout")
    return int(off.value), tuple(int(x) for x in shape)


def ttemb_forward(h: int, indices: int, offsets: int, nnz: int, batch: int, out: int, stream: int) -> int:
    return L.load().ttemb_forward(h, indices, offsets, int(nnz), int(batch), out, stream)


def ttemb_forward_weighted(h: int, indices: int, offsets: int, per_sample_weights: int, nnz: int,
                           batch: int, out: int, stream: int) -> int:
    return L.load().ttemb_forward_weighted(h, indices, offsets, per_sample_weights or None, int(nnz),
                                           int(batch), out, stream)


def ttemb_plan_batch(h: int, indices: int, offsets: int, per_sample_weights: int, nnz: int, batch: int,
               stream: int) -> int:
    return L.load().ttemb_plan_batch(h, indices, offsets, per_sample_weights or None, int(nnz), int(batch), stream)


def ttemb_forward_planned(h: int, out: int, stream: int) -> int:
    return L.load().ttemb_forward_planned(h, out, stream)


def ttemb_backward(h: int, grad_out: int, lr: float, stream: int) -> int:
    return L.load().ttemb_backward(h, grad_out, float(lr), stream)


def ttemb_update(h: int, lr: float, stream: int) -> int:
    return L.load().ttemb_update(h, float(lr), stream)


def ttemb_forward_host(h: int, indices: int, offsets: int, nnz: int, batch: int, out: int, stream: int) -> int:
    return L.load().ttemb_forward_host(h, indices, offsets, int(nnz), int(batch), out, stream)


def ttemb_backward_host(h: int, grad_out: int, lr: float, stream: int) -> int:
    return L.load().ttemb_backward_host(h, grad_out, float(lr), stream)


def ttemb_check(h: int, stream: int) -> int:
    return L.load().ttemb_check(h, stream)


def ttemb_get_plan(h: int) -> "L.ttemb_plan":
    p = L.ttemb_plan()
    check(L.load().ttemb_get_plan(h, C.byref(p)), "ttemb_get_plan")
    return p


def ttemb_read_counts(h: int, stream: int) -> Tuple[int, int, int, int]:
    v = (C.c_int64 * 4)()
    check(L.load().ttemb_read_counts(h, v, stream), "ttemb_read_counts")
    return tuple(int(x) for x in v)


def ttemb_set_timing(h: int, enable: bool) -> None:
    check(L.load().ttemb_set_timing(h, int(bool(enable))), "ttemb_set_timing")


def ttemb_stage_times(h: int) -> Dict[str, Tuple[float, int]]:
    n = 64
    ms = (C.c_double * n)()
    cnt = (C.c_int64 * n)()
    k = L.load().ttemb_stage_times(h, ms, cnt, n)
    if k < 0:
        raise TTEmbError(k, "ttemb_stage_times")
    return {ttemb_stage_name(i): (float(ms[i]), int(cnt[i])) for i in range(k)}


def ttemb_stage_name(i: int) -> str:
    return L.load().ttemb_stage_name(int(i)).decode()


def ttemb_set_bijection(h: int, bijection: int) -> None:
    check(L.load().ttemb_set_bijection(h, bijection or None), "ttemb_set_bijection")


def ttemb_total_rows(h: int) -> int:
    return int(L.load().ttemb_total_rows(h))


def ttemb_status_string(code: int) -> str:
    return L.status_string(code)


# ---------------------------------------------------------------------------
# Convenience owner
# ---------------------------------------------------------------------------
FLAT_ALIGN = 1024


class TTEmbeddingBag:
    """Table-batched TT-EmbeddingBag (sum pooling) on one CUDA device.

    Buffers (torch tensors, caller-owned in ABI terms): cores, state (Adagrad),
    grads, workspace.  Cores are zero until `load_cores` / `core_views` writes.
    """

    def __init__(self, table_rows, row_factors, col_factors, rank, max_batch, max_nnz,
                 optimizer: str = "sgd", adagrad_eps: float = 1e-10, fused_update: bool = False,
                 index_bits: int = 64, device: int = 0, fp32_cores: bool = False,
                 prefix_reuse: bool = True, aggregation: bool = True, mode: str = "sum",
                 dense: Sequence[bool] = ()):
        L.load()
        self.mode = mode
        self.dense = [bool(dense[t]) if len(dense) else False for t in range(len(table_rows))]
        self.table_rows = [int(x) for x in table_rows]
        self.row_factors = [tuple(int(y) for y in f) for f in row_factors]
        self.col_factors = tuple(int(x) for x in col_factors)
        self.rank = int(rank)
        self.T = len(self.table_rows)
        self.N = int(np.prod(self.col_factors))
        self.optimizer = optimizer
        self.fused = bool(fused_update)
        self.index_bits = int(index_bits)
        self.device = torch.device("cuda", device)
        self._cfg, self._tabs = make_config(table_rows, row_factors, col_factors, rank, max_batch,
                                            max_nnz, optimizer, adagrad_eps, fused_update, index_bits,
                                            fp32_cores=fp32_cores, prefix_reuse=prefix_reuse,
                                            aggregation=aggregation, mode=mode, dense=self.dense)
        cb, sb, gb, wb = ttemb_query_sizes(self._cfg)
        self.sizes = dict(core_bytes=cb, state_bytes=sb, grad_bytes=gb, workspace_bytes=wb)
        f32 = torch.float32
        # flat buffers padded to a multiple of FLAT_ALIGN floats, so a data-parallel group of up
        # to FLAT_ALIGN / 4 ranks can reduce-scatter / all-gather them in equal 16-byte-aligned
        # shards (the library only touches the first core_bytes; the padding stays 0)
        nfl = -(-(cb // 4) // FLAT_ALIGN) * FLAT_ALIGN
        self.n_floats = cb // 4
        self.cores = torch.zeros(nfl, dtype=f32, device=self.device)
        self.grads = torch.zeros(nfl, dtype=f32, device=self.device)
        self.state = torch.zeros(nfl, dtype=f32, device=self.device) if sb else None
        self.workspace = torch.empty(max(wb, 256), dtype=torch.uint8, device=self.device)
        self.h = ttemb_create(self._cfg, device, self.cores.data_ptr(),
                              self.state.data_ptr() if self.state is not None else 0,
                              self.grads.data_ptr(), self.workspace.data_ptr())
        self.layout = [[ttemb_core_layout(self.h, t, k) for k in range(3)] for t in range(self.T)]
        self.batch = 0
        self.nnz = 0

    @classmethod
    def from_config(cls, cfg, max_batch=None, max_nnz=None, **kw):
        B = cfg.batch if max_batch is None else max_batch
        nnz = B * cfg.num_tables * cfg.pooling if max_nnz is None else max_nnz
        kw.setdefault("dense", getattr(cfg, "dense", ()))
        return cls(cfg.table_rows, cfg.row_factors, cfg.col_factors, cfg.rank, B, nnz, **kw)

    def __del__(self):
        h = getattr(self, "h", None)
        if h:
            try:
                torch.cuda.synchronize(self.device)
                ttemb_destroy(h)
            except Exception:
                pass
            self.h = None

    # -- parameters --------------------------------------------------------
    def _views(self, buf: torch.Tensor):
        """Per table (C1, C2, C3) views at the configured rank; a zero-padded storage rank
        (ttemb_config.rank doc) is sliced away, so the views are strided then."""
        out = []
        R = self.rank
        for t in range(self.T):
            vs = []
            for k in range(3):
                off, shape = self.layout[t][k]
                shp = shape[:3] if k != 1 else shape
                if self.dense[t] and k == 0:
                    shp = shape[:2]            # hybrid: the plain table W[M][N]
                n = int(np.prod(shp))
                v = buf[off:off + n].view(*shp)
                if not self.dense[t]:
                    if k == 0:
                        v = v[:, :, :R]
                    elif k == 1:
                        v = v[:, :R, :, :R]
                    else:
                        v = v[:, :R, :]
                vs.append(v)
            out.append(tuple(vs))
        return out

    def core_views(self):
        return self._views(self.cores)

    def grad_views(self):
        return self._views(self.grads)

    def state_views(self):
        return self._views(self.state) if self.state is not None else None

    def load_cores(self, cores) -> None:
        """cores: per table (C1[m1][n1][R], C2[m2][R][n2][R], C3[m3][R][n3])."""
        for dst, src in zip(self.core_views(), cores):
            for d, s in zip(dst, src):
                d.copy_(torch.as_tensor(np.asarray(s, dtype=np.float32)).view(d.shape))

    # -- step ----------------------------------------------------------------
    def forward(self, indices: torch.Tensor, offsets: torch.Tensor, batch: int,
                out: Optional[torch.Tensor] = None, stream=None,
                per_sample_weights: Optional[torch.Tensor] = None) -> torch.Tensor:
        want = torch.int64 if self.index_bits == 64 else torch.int32
        assert indices.dtype == want and indices.is_cuda and offsets.dtype == torch.int64
        assert offsets.numel() == self.T * batch + 1
        if out is None:
            out = torch.empty(batch, self.T, self.N, dtype=torch.float32, device=self.device)
        nnz = indices.numel()
        psw = 0
        if per_sample_weights is not None:
            assert per_sample_weights.dtype == torch.float32 and per_sample_weights.is_cuda
            assert per_sample_weights.is_contiguous() and per_sample_weights.numel() == nnz
            psw = per_sample_weights.data_ptr() if nnz else 0
        rc = ttemb_forward_weighted(self.h, indices.data_ptr() if nnz else None, offsets.data_ptr(), psw,
                                    nnz, batch, out.data_ptr() if out.numel() else None, _stream_ptr(stream))
        check(rc, "ttemb_forward")
        self.batch, self.nnz = batch, nnz
        return out

    # -- cross-step pipelining: the index stage of the next batch on another stream ----------
    def sibling(self) -> "TTEmbeddingBag":
        """A second handle on the SAME cores / state / grads with its own workspace (plan), for
        running the next batch's index stage while this one computes (ttemb_plan_batch)."""
        other = object.__new__(TTEmbeddingBag)
        other.__dict__.update({k: v for k, v in self.__dict__.items() if k not in ("h", "workspace", "_bij")})
        other.workspace = torch.empty_like(self.workspace)
        other.h = ttemb_create(self._cfg, self.device.index, self.cores.data_ptr(),
                               self.state.data_ptr() if self.state is not None else 0,
                               self.grads.data_ptr(), other.workspace.data_ptr())
        if getattr(self, "_bij", None) is not None:
            other.set_bijection(self._bij)
        return other

    def plan_batch(self, indices: torch.Tensor, offsets: torch.Tensor, batch: int, stream=None,
                   per_sample_weights: Optional[torch.Tensor] = None) -> None:
        """Index stage only (ttemb_plan_batch); `offsets` must stay alive until forward_planned.
        (`plan()` returns a copy of the last plan's arrays.)"""
        nnz = indices.numel()
        psw = per_sample_weights.data_ptr() if (per_sample_weights is not None and nnz) else 0
        check(ttemb_plan_batch(self.h, indices.data_ptr() if nnz else None, offsets.data_ptr(), psw, nnz, batch,
                         _stream_ptr(stream)), "ttemb_plan_batch")
        self.batch, self.nnz = batch, nnz

    def forward_planned(self, out: Optional[torch.Tensor] = None, stream=None) -> torch.Tensor:
        if out is None:
            out = torch.empty(self.batch, self.T, self.N, dtype=torch.float32, device=self.device)
        check(ttemb_forward_planned(self.h, out.data_ptr() if out.numel() else None, _stream_ptr(stream)),
              "ttemb_forward_planned")
        return out

    def backward(self, grad_out: torch.Tensor, lr: float = 0.0, stream=None) -> None:
        assert grad_out.dtype == torch.float32 and grad_out.is_contiguous()
        assert tuple(grad_out.shape) == (self.batch, self.T, self.N)
        check(ttemb_backward(self.h, grad_out.data_ptr() if grad_out.numel() else None, lr,
                             _stream_ptr(stream)), "ttemb_backward")

    def update(self, lr: float, stream=None) -> None:
        check(ttemb_update(self.h, lr, _stream_ptr(stream)), "ttemb_update")

    def update_range(self, lr: float, begin: int, count: int, stream=None) -> None:
        """Optimizer step on floats [begin, begin + count) of the flat buffers (clipped to the
        library's part; the padding has no parameters)."""
        end = min(begin + count, self.n_floats)
        if end > begin:
            check(L.load().ttemb_update_range(self.h, lr, begin, end - begin, _stream_ptr(stream)),
                  "ttemb_update_range")

    def grad_buckets(self):
        """[(begin, count)] float ranges of the gradient buffer in the order the unfused backward
        finalises them (dense tables, C3 cores, C1 + C2 cores)."""
        b = (C.c_int64 * 3)()
        n = (C.c_int64 * 3)()
        k = L.load().ttemb_grad_buckets(self.h, b, n, 3)
        if k < 0:
            check(k, "ttemb_grad_buckets")
        return [(int(b[i]), int(n[i])) for i in range(k)]

    def set_bucket_events(self, events) -> None:
        """torch.cuda.Event objects (one per bucket) the backward records as buckets finish, or
        None.  The events are kept alive by this object."""
        self._bucket_events = list(events) if events else []
        for e in self._bucket_events:
            e.record(torch.cuda.current_stream(self.device))   # materialise the CUDA event handle
        arr = (C.c_void_p * 3)(*[e.cuda_event for e in self._bucket_events])
        check(L.load().ttemb_set_bucket_events(self.h, arr, len(self._bucket_events)), "ttemb_set_bucket_events")

    def forward_host(self, indices: torch.Tensor, offsets: torch.Tensor, batch: int,
                     out: torch.Tensor, stream=None) -> None:
        """indices / offsets / out in (pinned) host memory."""
        assert not indices.is_cuda and not offsets.is_cuda and not out.is_cuda
        nnz = indices.numel()
        check(ttemb_forward_host(self.h, indices.data_ptr() if nnz else None, offsets.data_ptr(), nnz,
                                 batch, out.data_ptr() if out.numel() else None, _stream_ptr(stream)),
              "ttemb_forward_host")
        self.batch, self.nnz = batch, nnz

    def backward_host(self, grad_out: torch.Tensor, lr: float = 0.0, stream=None) -> None:
        assert not grad_out.is_cuda
        check(ttemb_backward_host(self.h, grad_out.data_ptr() if grad_out.numel() else None, lr,
                                  _stream_ptr(stream)), "ttemb_backward_host")

    def check(self, stream=None) -> int:
        return ttemb_check(self.h, _stream_ptr(stream))

    def set_bijection(self, bijection: Optional[torch.Tensor]) -> None:
        """Runtime index bijection: a device tensor of sum(M_t) uint32 / int32 entries
        (table t's map at offset M_0 + ... + M_{t-1}), or None to switch it off.  The tensor is
        kept alive by this object."""
        if bijection is None:
            ttemb_set_bijection(self.h, 0)
            self._bij = None
            return
        assert bijection.is_cuda and bijection.dtype in (torch.int32, torch.uint32)
        assert bijection.is_contiguous() and bijection.numel() == ttemb_total_rows(self.h)
        self._bij = bijection
        ttemb_set_bijection(self.h, bijection.data_ptr())

    def counts(self, stream=None) -> Dict[str, int]:
        U, P, NG, err = ttemb_read_counts(self.h, _stream_ptr(stream))
        return dict(U=U, P=P, NG=NG, err=err)

    def all_counts(self, stream=None) -> Dict[str, int]:
        """Every device counter of the last forward's plan (include/ttemb.h ttemb_plan.counts):
        U, P, NG, error flags, multi-id-bag flag, Utt + 1, FFMA work units, split i2-groups."""
        torch.cuda.synchronize(self.device)
        p = ttemb_get_plan(self.h)
        v = _copy_device_u32(p.counts, 16, self.device).cpu().numpy().view("uint32")
        names = ("U", "P", "NG", "err", "multi", "utt1", "nchunks", "nsplit")
        return {k: int(v[i]) for i, k in enumerate(names)}

    def plan(self, stream=None) -> Dict[str, torch.Tensor]:
        """Copies of the index-stage outputs of the last forward (sizes from the counts)."""
        c = self.counts(stream)
        p = ttemb_get_plan(self.h)
        U, P, NG, nnz = c["U"], c["P"], c["NG"], int(p.nnz)
        size = {"skey": nnz, "spos": nnz, "bag_of": nnz, "inverse": nnz, "ukey": U, "seg_off": U + 1,
                "row_pfx": U, "row_i3": U, "pfx_t": P, "pfx_i1": P, "pfx_i2": P, "row_seg": P + 1,
                "grp_pfx": P, "grp_off": NG + 1, "grp_t": NG, "grp_i2": NG}
        out = {}
        for k, n in size.items():
            out[k] = _copy_device_u32(getattr(p, k), n, self.device)
        n1, n2, n3 = self.col_factors
        out["rows"] = _copy_device_f32(p.rows, U * self.N, self.device).view(U, self.N)
        out.update(U=U, P=P, NG=NG)
        return out

    # -- checkpoint / resume ---------------------------------------------------------------
    def _signature(self) -> Dict:
        return {"table_rows": list(self.table_rows), "row_factors": [list(f) for f in self.row_factors],
                "col_factors": list(self.col_factors), "rank": self.rank, "optimizer": self.optimizer,
                "dense": list(self.dense), "n_floats": self.n_floats}

    def state_dict(self) -> Dict:
        """Parameters and optimizer state as host tensors (a checkpoint): the flat core buffer
        (all tables, storage layout of ttemb_core_layout), the Adagrad accumulators if any, and
        the configuration they belong to.  Call between steps (the gradient buffer is not
        saved: it is zero after an update / a fused backward)."""
        torch.cuda.synchronize(self.device)
        sd = {"format": "ttemb-v1", "config": self._signature(),
              "cores": self.cores[:self.n_floats].detach().cpu().clone()}
        if self.state is not None:
            sd["state"] = self.state[:self.n_floats].detach().cpu().clone()
        return sd

    def load_state_dict(self, sd: Dict) -> None:
        """Restore a state_dict() of an identically configured instance (bitwise)."""
        if sd.get("format") != "ttemb-v1" or sd.get("config") != self._signature():
            raise ValueError("checkpoint does not match this TTEmbeddingBag's configuration")
        if (self.state is None) != ("state" not in sd):
            raise ValueError("checkpoint optimizer state does not match")
        self.cores[:self.n_floats].copy_(sd["cores"].to(self.device))
        if self.state is not None:
            self.state[:self.n_floats].copy_(sd["state"].to(self.device))
        self.grads.zero_()
        torch.cuda.synchronize(self.device)

    def set_timing(self, enable: bool) -> None:
        ttemb_set_timing(self.h, enable)

    def stage_times(self) -> Dict[str, Tuple[float, int]]:
        return ttemb_stage_times(self.h)


class _DevArray:
    """A raw device pointer exposed through __cuda_array_interface__ (zero-copy view)."""

    def __init__(self, ptr: int, n: int, typestr: str):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": typestr, "data": (ptr, False),
                                         "version": 2}


def _copy_device_u32(ptr: int, n: int, device) -> torch.Tensor:
    if n <= 0:
        return torch.empty(0, dtype=torch.int32, device=device)
    return torch.as_tensor(_DevArray(ptr, n, "<u4"), device=device).view(torch.int32).clone()


def _copy_device_f32(ptr: int, n: int, device) -> torch.Tensor:
    if n <= 0:
        return torch.empty(0, dtype=torch.float32, device=device)
    return torch.as_tensor(_DevArray(ptr, n, "<f4"), device=device).clone()


class HostStepPipeline:
    """End-to-end training steps from pinned host memory with the copies overlapped.

    step(k): the inputs of step k (ids, offsets, grad_out; pinned host tensors) are copied to a
    device staging slot on an H2D stream while the previous step computes; forward + backward
    (the library's kernels) run on the compute stream once the slot has landed; the pooled
    output is copied back to the caller's pinned host tensor on a D2H stream while the next step
    computes.  `depth` slots rotate; a slot is refilled only after its last step's compute and
    output copy finished (events), so nothing is overwritten in flight.  Host tensors must not be
    modified until `wait(k)` returned for the step that uses them.
    """

    def __init__(self, emb: "TTEmbeddingBag", max_nnz: int, batch: int, depth: int = 2):
        self.emb, self.depth, self.B = emb, int(depth), int(batch)
        dev = emb.device
        it = torch.int64 if emb.index_bits == 64 else torch.int32
        self.h2d = torch.cuda.Stream(device=dev)
        self.d2h = torch.cuda.Stream(device=dev)
        self.idx = [torch.empty(max(max_nnz, 1), dtype=it, device=dev) for _ in range(depth)]
        self.off = [torch.empty(emb.T * batch + 1, dtype=torch.int64, device=dev) for _ in range(depth)]
        self.grad = [torch.empty(batch, emb.T, emb.N, dtype=torch.float32, device=dev) for _ in range(depth)]
        self.out = [torch.empty(batch, emb.T, emb.N, dtype=torch.float32, device=dev) for _ in range(depth)]
        self.ev_in = [torch.cuda.Event() for _ in range(depth)]
        self.ev_comp = [torch.cuda.Event() for _ in range(depth)]
        self.ev_out = [torch.cuda.Event() for _ in range(depth)]
        self.k = 0

    def step(self, h_idx: torch.Tensor, h_off: torch.Tensor, h_grad: torch.Tensor, h_out: torch.Tensor,
             lr: float) -> int:
        """Enqueue one training step; returns its step number (for wait)."""
        k, s = self.k, self.k % self.depth
        comp = torch.cuda.current_stream(self.emb.device)
        nnz = h_idx.numel()
        if k >= self.depth:
            self.h2d.wait_event(self.ev_comp[s])          # the slot's inputs were consumed
            comp.wait_event(self.ev_out[s])               # the slot's output was copied out
        with torch.cuda.stream(self.h2d):
            self.idx[s][:nnz].copy_(h_idx, non_blocking=True)
            self.off[s].copy_(h_off, non_blocking=True)
            self.grad[s].copy_(h_grad, non_blocking=True)
            self.ev_in[s].record(self.h2d)
        comp.wait_event(self.ev_in[s])
        self.emb.forward(self.idx[s][:nnz], self.off[s], self.B, out=self.out[s], stream=comp)
        self.emb.backward(self.grad[s], lr=lr, stream=comp)
        self.ev_comp[s].record(comp)
        self.d2h.wait_event(self.ev_comp[s])
        with torch.cuda.stream(self.d2h):
            h_out.copy_(self.out[s], non_blocking=True)
            self.ev_out[s].record(self.d2h)
        self.k += 1
        return k

    def wait(self, k: int) -> None:
        """Block until step k's output reached host memory."""
        self.ev_out[k % self.depth].synchronize()
