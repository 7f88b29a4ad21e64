"""ctypes wrapper around the C oracle (oracle/ttemb_oracle.c).

TEST INFRASTRUCTURE ONLY: imported by tests/, __graft_entry__.smoke() and
bench.py's cpu_baseline / --impl reference legs.  The product package
(paper_conf_sc_wangwfmmd22_b200) never imports this module, and this module
never imports the product package.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
from typing import List, Sequence, Tuple

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ttemb_oracle.c")
_LIB = os.path.join(_HERE, "libttemb_oracle.so")
_lib = None

ERR_INVALID = -1
ERR_INDEX_RANGE = -3


def build(force: bool = False) -> str:
    """Compile the oracle (gcc, -O2, OpenMP, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < max(
            os.path.getmtime(_SRC), os.path.getmtime(os.path.join(_HERE, "ttemb_oracle.h"))):
        cmd = ["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared", "-fno-fast-math",
               "-ffp-contract=off", "-o", _LIB + ".tmp", _SRC, "-lm"]
        subprocess.check_call(cmd, cwd=_HERE)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


class _Shape(C.Structure):
    _fields_ = [("T", C.c_int32), ("rows", C.POINTER(C.c_int64)), ("mfac", C.POINTER(C.c_int32)),
                ("n", C.c_int32 * 3), ("R", C.c_int32), ("dense", C.POINTER(C.c_int32))]


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        u32p = C.POINTER(C.c_uint32)
        i64p = C.POINTER(C.c_int64)
        _lib.ttref_plan.argtypes = [C.POINTER(_Shape), i64p, i64p, C.c_int64, C.c_int32] + [u32p] * 16 + [i64p]
        _lib.ttref_forward.argtypes = [C.POINTER(_Shape), C.c_void_p, C.c_void_p, C.c_void_p, i64p, i64p,
                                       C.c_int64, C.c_int32, C.c_int, C.POINTER(C.c_double)]
        _lib.ttref_backward.argtypes = [C.POINTER(_Shape), C.c_void_p, C.c_void_p, C.c_void_p, i64p, i64p,
                                        C.c_int64, C.c_int32, C.POINTER(C.c_float), C.c_int,
                                        C.c_void_p, C.c_void_p, C.c_void_p]
        _lib.ttref_forward_ex.argtypes = [C.POINTER(_Shape), C.c_void_p, C.c_void_p, C.c_void_p, i64p, i64p,
                                          C.c_int64, C.c_int32, C.POINTER(C.c_float), C.c_int, C.c_int,
                                          C.POINTER(C.c_double)]
        _lib.ttref_backward_ex.argtypes = [C.POINTER(_Shape), C.c_void_p, C.c_void_p, C.c_void_p, i64p, i64p,
                                           C.c_int64, C.c_int32, C.POINTER(C.c_float), C.c_int,
                                           C.POINTER(C.c_float), C.c_int, C.c_void_p, C.c_void_p, C.c_void_p]
        _lib.ttref_update.argtypes = [C.c_int, C.c_double, C.c_double, C.c_int64, C.POINTER(C.c_float),
                                      C.POINTER(C.c_float), C.POINTER(C.c_double)]
        _lib.ttref_digits.argtypes = [C.POINTER(C.c_int32), C.c_int64, C.POINTER(C.c_int64)]
        _lib.ttref_row_chain.argtypes = [C.POINTER(_Shape), C.c_int, C.POINTER(C.c_float), C.POINTER(C.c_float),
                                         C.POINTER(C.c_float), C.c_int64, C.POINTER(C.c_double)]
        _lib.ttref_row_literal.argtypes = _lib.ttref_row_chain.argtypes
        _lib.ttref_num_threads.restype = C.c_int
        _lib.ttref_apply_bijection.argtypes = [C.POINTER(_Shape), C.c_void_p, i64p, i64p, C.c_int64,
                                               C.c_int32, i64p]
    return _lib


def _p(a, ct):
    return a.ctypes.data_as(C.POINTER(ct))


class OracleError(RuntimeError):
    def __init__(self, code):
        super().__init__(f"oracle status {code}")
        self.code = code


class Oracle:
    """fp64 oracle for one table set (shared N = n1 n2 n3 and rank R)."""

    def __init__(self, table_rows: Sequence[int], row_factors: Sequence[Tuple[int, int, int]],
                 col_factors: Tuple[int, int, int], rank: int, dense: Sequence[bool] = ()):
        """dense[t] = table t kept uncompressed (hybrid placement): its cores are
        (W[M][N], empty, empty)."""
        self.rows = np.ascontiguousarray(table_rows, dtype=np.int64)
        self.mfac = np.ascontiguousarray(row_factors, dtype=np.int32).reshape(-1, 3)
        self.n = tuple(int(x) for x in col_factors)
        self.R = int(rank)
        self.T = len(self.rows)
        self.N = self.n[0] * self.n[1] * self.n[2]
        self.dense = np.ascontiguousarray([1 if d else 0 for d in dense] if len(dense) else [0] * self.T,
                                          dtype=np.int32)
        self._shape = _Shape(self.T, _p(self.rows, C.c_int64), _p(self.mfac, C.c_int32),
                             (C.c_int32 * 3)(*self.n), self.R, _p(self.dense, C.c_int32))

    @classmethod
    def from_config(cls, cfg):
        return cls(cfg.table_rows, cfg.row_factors, cfg.col_factors, cfg.rank, getattr(cfg, "dense", ()))

    @staticmethod
    def num_threads() -> int:
        return int(lib().ttref_num_threads())

    # -- helpers -----------------------------------------------------------
    def digits(self, t: int, row: int) -> Tuple[int, int, int]:
        d = np.zeros(3, np.int64)
        lib().ttref_digits(_p(self.mfac[t].copy(), C.c_int32), int(row), _p(d, C.c_int64))
        return tuple(int(x) for x in d)

    def row(self, cores, t: int, row: int, literal: bool = False) -> np.ndarray:
        c1, c2, c3 = (np.ascontiguousarray(x, dtype=np.float32) for x in cores[t])
        e = np.zeros(self.N, np.float64)
        f = lib().ttref_row_literal if literal else lib().ttref_row_chain
        f(C.byref(self._shape), int(t), _p(c1, C.c_float), _p(c2, C.c_float), _p(c3, C.c_float),
          int(row), _p(e, C.c_double))
        return e

    def _core_ptrs(self, cores, k):
        arrs = [np.ascontiguousarray(c[k], dtype=np.float32) for c in cores]
        ptrs = (C.c_void_p * self.T)(*[a.ctypes.data for a in arrs])
        return arrs, ptrs

    @staticmethod
    def _ids(indices, offsets):
        return (np.ascontiguousarray(indices, dtype=np.int64),
                np.ascontiguousarray(offsets, dtype=np.int64))

    def apply_bijection(self, bijection, indices, offsets, batch: int) -> np.ndarray:
        """New_Batch = { index_t(i_j) }; bijection: per table an int array [M_t]."""
        idx, off = self._ids(indices, offsets)
        maps = [np.ascontiguousarray(b, dtype=np.int64) for b in bijection]
        assert len(maps) == self.T
        ptrs = (C.c_void_p * self.T)(*[m.ctypes.data for m in maps])
        out = np.zeros(max(len(idx), 1), np.int64)
        rc = lib().ttref_apply_bijection(C.byref(self._shape), ptrs, _p(idx, C.c_int64),
                                         _p(off, C.c_int64), len(idx), int(batch), _p(out, C.c_int64))
        if rc:
            raise OracleError(rc)
        return out[:len(idx)]

    # -- plan --------------------------------------------------------------
    def plan(self, indices, offsets, batch: int) -> dict:
        idx, off = self._ids(indices, offsets)
        nnz = len(idx)
        n = max(nnz, 1)
        names = ["skey", "spos", "bag_of", "ukey", "seg_off", "inverse", "row_pfx", "row_i3",
                 "pfx_t", "pfx_i1", "pfx_i2", "row_seg", "grp_pfx", "grp_off", "grp_t", "grp_i2"]
        arr = {k: np.zeros(n + 1, np.uint32) for k in names}
        counts = np.zeros(3, np.int64)
        rc = lib().ttref_plan(C.byref(self._shape), _p(idx, C.c_int64), _p(off, C.c_int64), nnz,
                              int(batch), *[_p(arr[k], C.c_uint32) for k in names],
                              _p(counts, C.c_int64))
        if rc:
            raise OracleError(rc)
        U, P, NG = (int(x) for x in counts)
        size = {"skey": nnz, "spos": nnz, "bag_of": nnz, "inverse": nnz, "ukey": U, "seg_off": U + 1,
                "row_pfx": U, "row_i3": U, "pfx_t": P, "pfx_i1": P, "pfx_i2": P, "row_seg": P + 1,
                "grp_pfx": P, "grp_off": NG + 1, "grp_t": NG, "grp_i2": NG}
        out = {k: arr[k][:size[k]].copy() for k in names}
        out.update(U=U, P=P, NG=NG)
        return out

    # -- forward / backward ------------------------------------------------
    @staticmethod
    def _mode(mode: str) -> int:
        return {"sum": 0, "mean": 1}[mode]

    def forward(self, cores, indices, offsets, batch: int, literal: bool = False,
                absolute: bool = False, per_sample_weights=None, mode: str = "sum") -> np.ndarray:
        """out[B][T][N] fp64.  absolute=True evaluates the |C| (and |weights|) companion.
        mode / per_sample_weights follow nn.EmbeddingBag (weights only with mode="sum")."""
        if absolute:
            cores = [tuple(np.abs(x) for x in c) for c in cores]
        idx, off = self._ids(indices, offsets)
        psw = None
        if per_sample_weights is not None:
            psw = np.ascontiguousarray(per_sample_weights, dtype=np.float32)
            if absolute:
                psw = np.abs(psw)
        k1, p1 = self._core_ptrs(cores, 0)
        k2, p2 = self._core_ptrs(cores, 1)
        k3, p3 = self._core_ptrs(cores, 2)
        out = np.zeros((batch, self.T, self.N), np.float64)
        rc = lib().ttref_forward_ex(C.byref(self._shape), p1, p2, p3, _p(idx, C.c_int64),
                                    _p(off, C.c_int64), len(idx), int(batch),
                                    _p(psw, C.c_float) if psw is not None else None, self._mode(mode),
                                    int(literal), _p(out, C.c_double))
        if rc:
            raise OracleError(rc)
        return out

    def backward(self, cores, indices, offsets, batch: int, grad_out, literal: bool = False,
                 absolute: bool = False, per_sample_weights=None,
                 mode: str = "sum") -> List[Tuple[np.ndarray, np.ndarray, np.ndarray]]:
        """Core gradients of L = sum(out * grad_out), fp64, per table (dC1, dC2, dC3).
        absolute=True evaluates the |C|, |grad_out| (|weights|) companion."""
        go = np.ascontiguousarray(grad_out, dtype=np.float32)
        psw = None
        if per_sample_weights is not None:
            psw = np.ascontiguousarray(per_sample_weights, dtype=np.float32)
            if absolute:
                psw = np.abs(psw)
        if absolute:
            cores = [tuple(np.abs(x) for x in c) for c in cores]
            go = np.abs(go)
        assert go.shape == (batch, self.T, self.N)
        idx, off = self._ids(indices, offsets)
        k1, p1 = self._core_ptrs(cores, 0)
        k2, p2 = self._core_ptrs(cores, 1)
        k3, p3 = self._core_ptrs(cores, 2)
        grads = [tuple(np.zeros(np.shape(c[k]), np.float64) for k in range(3)) for c in cores]
        g1 = (C.c_void_p * self.T)(*[g[0].ctypes.data for g in grads])
        g2 = (C.c_void_p * self.T)(*[g[1].ctypes.data for g in grads])
        g3 = (C.c_void_p * self.T)(*[g[2].ctypes.data for g in grads])
        rc = lib().ttref_backward_ex(C.byref(self._shape), p1, p2, p3, _p(idx, C.c_int64), _p(off, C.c_int64),
                                     len(idx), int(batch), _p(psw, C.c_float) if psw is not None else None,
                                     self._mode(mode), _p(go, C.c_float), int(literal), g1, g2, g3)
        if rc:
            raise OracleError(rc)
        return grads

    @staticmethod
    def update(opt: str, lr: float, param: np.ndarray, grad: np.ndarray, state: np.ndarray = None,
               eps: float = 1e-10):
        """Returns (new_param float32, new_state float32 or None); inputs untouched."""
        p = np.ascontiguousarray(param, dtype=np.float32).copy()
        g = np.ascontiguousarray(grad, dtype=np.float64)
        o = {"sgd": 0, "adagrad": 1}[opt]
        s = None
        if o == 1:
            s = (np.zeros_like(p) if state is None else np.ascontiguousarray(state, np.float32).copy())
        rc = lib().ttref_update(o, float(lr), float(eps), p.size, _p(p, C.c_float),
                                _p(s, C.c_float) if s is not None else None, _p(g, C.c_double))
        if rc:
            raise OracleError(rc)
        return p, s
