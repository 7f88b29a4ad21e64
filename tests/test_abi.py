"""C-ABI checks that need no GPU: the library loads, exports every symbol that
include/ttemb.h declares, and the host-side validation / sizing behaves."""
import ctypes as C
import os
import re
import subprocess

import pytest

import paper_conf_sc_wangwfmmd22_b200 as tt
from paper_conf_sc_wangwfmmd22_b200 import _lib as L
from synth import workload as W

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "ttemb.h")


def declared_symbols():
    src = open(HEADER).read()
    return sorted(set(re.findall(r"^\s*(?:int|uint64_t|const char\*)\s+(ttemb_\w+)\s*\(", src, re.M)))


def test_header_symbols_exported():
    syms = declared_symbols()
    assert len(syms) >= 15
    out = subprocess.check_output(["nm", "-D", "--defined-only", L.LIB_PATH]).decode()
    exported = set(re.findall(r"\bT (ttemb_\w+)", out))
    missing = [s for s in syms if s not in exported]
    assert not missing, missing
    assert set(L.SYMBOLS) == set(syms)
    lib = L.load()
    for s in syms:
        assert getattr(lib, s) is not None


def test_library_is_sm100a():
    out = subprocess.check_output(["/usr/local/cuda/bin/cuobjdump", "--list-elf", L.LIB_PATH]).decode()
    assert "sm_100a" in out


def test_oracle_not_linked_into_product():
    out = subprocess.check_output(["nm", "-D", L.LIB_PATH]).decode()
    assert "ttref_" not in out
    # no product source imports or includes the oracle
    for d, _, fs in os.walk(os.path.join(ROOT, "paper_conf_sc_wangwfmmd22_b200")):
        for f in fs:
            if f.endswith((".py", ".cu", ".cuh", ".h")):
                s = open(os.path.join(d, f)).read()
                assert not re.search(r"^\s*(import oracle|from oracle|#include .*ttemb_oracle)", s, re.M)


def _cfg(**kw):
    c = W.config("c2")
    args = dict(table_rows=c.table_rows, row_factors=c.row_factors, col_factors=c.col_factors,
                rank=c.rank, max_batch=c.batch, max_nnz=c.batch * c.num_tables)
    args.update(kw)
    return tt.make_config(**args)


def test_query_sizes_consistent():
    cfg, keep = _cfg(fp32_cores=True)     # (the tensor-core path stores R = 16 zero-padded to 32)
    core, state, grad, ws = tt.ttemb_query_sizes(cfg)
    c = W.config("c2")
    assert core == grad and state == 0 and ws > 0
    # padded per-table blocks: at least the exact core bytes, at most 16 B per block more
    assert W.core_bytes(c) <= core <= W.core_bytes(c) + 16 * 3 * c.num_tables
    cfg2, keep2 = _cfg(optimizer="adagrad", fp32_cores=True)
    assert tt.ttemb_query_sizes(cfg2)[1] == core


@pytest.mark.parametrize("kw,code", [
    (dict(num_cores=4), L.TTEMB_ERR_UNSUPPORTED),
    (dict(rank=0), L.TTEMB_ERR_INVALID_ARG),
    (dict(rank=129), L.TTEMB_ERR_UNSUPPORTED),
    (dict(index_bits=16), L.TTEMB_ERR_INVALID_ARG),
    (dict(row_factors=[(1, 1, 1)] * 20), L.TTEMB_ERR_INVALID_ARG),     # prod < M
    (dict(max_nnz=(1 << 30) + 1), L.TTEMB_ERR_UNSUPPORTED),
    (dict(table_rows=[0] + list(W.config("c2").table_rows[1:])), L.TTEMB_ERR_INVALID_ARG),
    (dict(optimizer="adagrad", adagrad_eps=0.0), L.TTEMB_ERR_INVALID_ARG),   # 0/0 on padding
    (dict(max_batch=1 << 23), L.TTEMB_ERR_UNSUPPORTED),                    # T B dim >= 2^31 elements
])
def test_query_sizes_rejects(kw, code):
    cfg, keep = _cfg(**kw)
    v = [C.c_size_t() for _ in range(4)]
    rc = L.load().ttemb_query_sizes(C.byref(cfg), *[C.byref(x) for x in v])
    assert rc == code


def test_bad_dim_rejected():
    cfg, keep = _cfg()
    cfg.dim = 17
    v = [C.c_size_t() for _ in range(4)]
    assert L.load().ttemb_query_sizes(C.byref(cfg), *[C.byref(x) for x in v]) == L.TTEMB_ERR_INVALID_ARG


def test_null_handle_calls_fail_cleanly():
    lib = L.load()
    assert lib.ttemb_forward(None, None, None, 0, 0, None, None) == L.TTEMB_ERR_INVALID_ARG
    assert lib.ttemb_backward(None, None, 0.0, None) == L.TTEMB_ERR_INVALID_ARG
    assert lib.ttemb_update(None, 0.0, None) == L.TTEMB_ERR_INVALID_ARG
    assert lib.ttemb_destroy(None) == L.TTEMB_ERR_INVALID_ARG
    assert tt.ttemb_status_string(-3) == "index out of range"
    assert tt.ttemb_stage_name(9) == "fwd_prefix"


def test_create_rejects_null_buffers():
    cfg, keep = _cfg()
    h = C.c_void_p()
    rc = L.load().ttemb_create(C.byref(cfg), 0, None, None, None, None, C.byref(h))
    assert rc == L.TTEMB_ERR_INVALID_ARG and not h.value


def test_ablation_flags_accepted_and_size_the_workspace():
    """TTEMB_NO_PREFIX_REUSE / TTEMB_NO_AGGREGATION are valid flags; they only grow
    the workspace (U capacity = nnz, P capacity = U); unknown flag bits are rejected."""
    base = tt.ttemb_query_sizes(_cfg()[0])
    for kw in (dict(prefix_reuse=False), dict(aggregation=False), dict(prefix_reuse=False, aggregation=False)):
        cfg, keep = _cfg(**kw)
        core, state, grad, ws = tt.ttemb_query_sizes(cfg)
        assert (core, state, grad) == base[:3] and ws >= base[3]
    cfg, keep = _cfg()
    cfg.flags = 1 << 7
    v = [C.c_size_t() for _ in range(4)]
    assert L.load().ttemb_query_sizes(C.byref(cfg), *[C.byref(x) for x in v]) == L.TTEMB_ERR_INVALID_ARG


def test_hybrid_tables_sizes_and_layout_validation():
    """Hybrid placement: a dense table's factors are ignored and it occupies M x dim floats;
    the core / grad buffers grow by exactly the dense tables' size (16-byte padded blocks)."""
    c = W.config("c2")
    h = W.hybrid(c)
    cfg_tt, k1 = _cfg(fp32_cores=True)
    cfg_h, k2 = tt.make_config(h.table_rows, [(0, 0, 0) if d else f for d, f in zip(h.dense, h.row_factors)],
                               h.col_factors, h.rank, h.batch, h.batch * h.num_tables, dense=h.dense,
                               fp32_cores=True)   # (unpadded rank: exact byte count)
    core_h = tt.ttemb_query_sizes(cfg_h)[0]
    assert W.core_bytes(h) <= core_h <= W.core_bytes(h) + 16 * 3 * h.num_tables
    assert core_h != tt.ttemb_query_sizes(cfg_tt)[0]
