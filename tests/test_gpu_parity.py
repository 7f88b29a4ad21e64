"""CUDA path (libttemb.so through the C ABI) vs the CPU oracle, element by element.

Integer plan: bit-exact.  Floats: |gpu - oracle| <= tol * oracle(|inputs|) with
tol = 1e-5 for the forward output and 1e-4 for core gradients (BASELINE.json
north_star).  The oracle never sees a value produced
by the CUDA path.
"""
import numpy as np
import pytest
import torch

from oracle import Oracle
from synth import workload as W
from tests.helpers import assert_companion, assert_update_close, plan_key

pytestmark = pytest.mark.gpu

if torch.cuda.is_available():
    import paper_conf_sc_wangwfmmd22_b200 as tt
    from paper_conf_sc_wangwfmmd22_b200 import _lib as L

DEV = torch.device("cuda", 0)


def gpu_emb(cfg, B, nnz, **kw):
    kw.setdefault("dense", getattr(cfg, "dense", ()))
    emb = tt.TTEmbeddingBag(cfg.table_rows, cfg.row_factors, cfg.col_factors, cfg.rank,
                            max(B, 1), max(nnz, 1), **kw)
    return emb


def run_forward(emb, idx, off, B, index_bits=64):
    it = torch.as_tensor(idx.astype(np.int64 if index_bits == 64 else np.int32), device=DEV)
    ot = torch.as_tensor(off, device=DEV)
    out = emb.forward(it, ot, B)
    return out


def check_plan(emb, orc, idx, off, B):
    mine = emb.plan()
    ref = orc.plan(idx, off, B)
    for k in ("U", "P", "NG"):
        assert mine[k] == ref[k], (k, mine[k], ref[k])
    for k, v in ref.items():
        if isinstance(v, np.ndarray):
            got = mine[k].cpu().numpy().view(np.uint32)
            np.testing.assert_array_equal(got, v, err_msg=k)
    return mine, ref


def small_cases():
    return [
        ("c1", W.config("c1"), None),
        ("multi-var-L", W.small_config([37, 100, 5, 1000], [(3, 4, 4), (5, 4, 5), (1, 2, 3), (10, 10, 10)],
                                       (2, 3, 2), 5, 33, 1, 1.05), "var"),
        ("r1-kron", W.small_config([60], [(3, 4, 5)], (2, 3, 2), 1, 17, 3), None),
        ("dup-heavy", W.small_config([50], [(2, 5, 5)], (2, 2, 2), 4, 40, 7, 2.0), None),
        ("wide-R128", W.small_config([3000, 200], [(15, 15, 15), (6, 6, 6)], (4, 4, 8), 128, 24, 2, 1.05), None),
        ("odd-dims", W.small_config([777], [(9, 10, 9)], (3, 1, 5), 7, 50, 2, 1.1), "var"),
        # R = 64 (tensor-core path): n1 = 2 / 4 / 8, n3 = 4 / 8, hot groups spanning m-tiles
        ("tc-n1-2", W.small_config([20000, 300], [(28, 28, 26), (7, 7, 7)], (2, 2, 4), 64, 96, 3, 1.05), "var"),
        ("tc-n1-8-n3-8", W.small_config([5000], [(18, 18, 16)], (8, 1, 8), 64, 64, 2, 1.2), None),
        ("tc-multitile", W.small_config([400000], [(74, 74, 74)], (4, 4, 8), 64, 512, 4, 0.6), None),
        ("tc-mixedmag", W.small_config([3000, 900], [(15, 15, 14), (10, 10, 9)], (4, 2, 4), 64, 80, 2, 1.05), "mixed"),
    ]


def make_inputs(cfg, mode, seed=0, batch=None):
    B = cfg.batch if batch is None else batch
    lens = None
    if mode == "var" or mode == "mixed":
        rng = np.random.default_rng(seed)
        lens = rng.integers(0, 6, size=cfg.num_tables * B)
        lens[0] = 0
        lens[-1] = 0
    idx, off = W.make_batch(cfg, step=seed, seed=seed, batch=B, lengths=lens)
    return idx, off, B


# ---------------------------------------------------------------------------
@pytest.mark.parametrize("name,cfg,mode", small_cases(), ids=[c[0] for c in small_cases()])
def test_forward_backward_small(name, cfg, mode):
    idx, off, B = make_inputs(cfg, mode, seed=3)
    cores = W.make_cores(cfg, seed=3, mixed_magnitude=(mode == "mixed"))
    go = W.make_grad_out(cfg, B, seed=3)
    emb = gpu_emb(cfg, B, len(idx))
    emb.load_cores(cores)
    out = run_forward(emb, idx, off, B)
    emb.backward(torch.as_tensor(go, device=DEV))
    assert emb.check() == 0
    orc = Oracle.from_config(cfg)
    check_plan(emb, orc, idx, off, B)
    ref = orc.forward(cores, idx, off, B)
    ref_abs = orc.forward(cores, idx, off, B, absolute=True)
    assert_companion(out.cpu().numpy(), ref, ref_abs, 1e-5, "forward")
    g = orc.backward(cores, idx, off, B, go)
    ga = orc.backward(cores, idx, off, B, go, absolute=True)
    for t, mine in enumerate(emb.grad_views()):
        for k in range(3):
            assert_companion(mine[k].cpu().numpy(), g[t][k], ga[t][k], 1e-4, f"dC{k+1} table {t}")


@pytest.mark.parametrize("name", ["c1", "c2", "c3"])
def test_configs_full_batch(name):
    cfg = W.config(name)
    idx, off = W.make_batch(cfg, seed=7)
    B = cfg.batch
    cores = W.make_cores(cfg, seed=7)
    go = W.make_grad_out(cfg, B, seed=7)
    emb = gpu_emb(cfg, B, len(idx))
    emb.load_cores(cores)
    out = run_forward(emb, idx, off, B)
    emb.backward(torch.as_tensor(go, device=DEV))
    assert emb.check() == 0
    orc = Oracle.from_config(cfg)
    check_plan(emb, orc, idx, off, B)
    assert_companion(out.cpu().numpy(), orc.forward(cores, idx, off, B),
                     orc.forward(cores, idx, off, B, absolute=True), 1e-5, "forward")
    g = orc.backward(cores, idx, off, B, go)
    ga = orc.backward(cores, idx, off, B, go, absolute=True)
    for t, mine in enumerate(emb.grad_views()):
        for k in range(3):
            assert_companion(mine[k].cpu().numpy(), g[t][k], ga[t][k], 1e-4, f"dC{k+1} t{t}")


@pytest.mark.parametrize("fp32_cores", [False, True], ids=["tcgen05", "fp32-cores"])
def test_c4_reduced_batch(fp32_cores):
    """Criteo-TB shape (26 tables, R=64, N=64) at batch 2048: every output checked, on the
    tensor-core (3xTF32) path and on the FP32 CUDA-core path."""
    cfg = W.config("c4")
    B = 2048
    idx, off = W.make_batch(cfg, seed=11, batch=B)
    cores = W.make_cores(cfg, seed=11)
    go = W.make_grad_out(cfg, B, seed=11)
    emb = gpu_emb(cfg, B, len(idx), fp32_cores=fp32_cores)
    emb.load_cores(cores)
    out = run_forward(emb, idx, off, B)
    emb.backward(torch.as_tensor(go, device=DEV))
    orc = Oracle.from_config(cfg)
    check_plan(emb, orc, idx, off, B)
    assert_companion(out.cpu().numpy(), orc.forward(cores, idx, off, B),
                     orc.forward(cores, idx, off, B, absolute=True), 1e-5, "forward")
    g = orc.backward(cores, idx, off, B, go)
    ga = orc.backward(cores, idx, off, B, go, absolute=True)
    for t, mine in enumerate(emb.grad_views()):
        for k in range(3):
            assert_companion(mine[k].cpu().numpy(), g[t][k], ga[t][k], 1e-4, f"dC{k+1} t{t}")


def _sub_batch(off, keep):
    """Offsets of the batch restricted to the positions in `keep` (bags keep their slot)."""
    lens = np.diff(off)
    bag = np.repeat(np.arange(len(lens)), lens)
    nl = np.bincount(bag[keep], minlength=len(lens))
    return np.concatenate([[0], np.cumsum(nl)]).astype(np.int64)


def _check_plan_full(emb, cfg, idx, off, B):
    plan = emb.plan()
    key = plan_key(cfg, idx, off, B)
    uk, inv = np.unique(key, return_inverse=True)
    assert plan["U"] == len(uk)
    np.testing.assert_array_equal(plan["ukey"].cpu().numpy().view(np.uint32), uk)
    np.testing.assert_array_equal(plan["inverse"].cpu().numpy().view(np.uint32), inv)


@pytest.mark.parametrize("opt", ["sgd", "adagrad"])
def test_c4_full_batch(opt):
    """Criteo-TB shape at the bench batch (B = 16384, 26 tables, R = 64) in the bench launch
    configuration: plan bit-exact vs numpy; the WHOLE forward output and every core gradient
    (unfused) vs the oracle on the full batch; the fused update (the bench's mode) vs the oracle
    update of the oracle gradients, every slice of every table."""
    cfg = W.config("c4")
    B = cfg.batch
    idx, off = W.make_batch(cfg, seed=5, batch=B)
    cores = W.make_cores(cfg, seed=5)
    go = W.make_grad_out(cfg, B, seed=5)
    orc = Oracle.from_config(cfg)
    g = orc.backward(cores, idx, off, B, go)
    ga = orc.backward(cores, idx, off, B, go, absolute=True)
    lr = 0.05
    if opt == "sgd":
        emb = gpu_emb(cfg, B, len(idx))
        emb.load_cores(cores)
        out = run_forward(emb, idx, off, B).cpu().numpy()
        assert emb.check() == 0
        _check_plan_full(emb, cfg, idx, off, B)
        assert_companion(out, orc.forward(cores, idx, off, B), orc.forward(cores, idx, off, B, absolute=True),
                         1e-5, "c4 forward")
        emb.backward(torch.as_tensor(go, device=DEV))
        for t, mine in enumerate(emb.grad_views()):
            for k in range(3):
                assert_companion(mine[k].cpu().numpy(), g[t][k], ga[t][k], 1e-4, f"c4 dC{k+1} t{t}")
        del emb
    emb = gpu_emb(cfg, B, len(idx), optimizer=opt, fused_update=True)
    emb.load_cores(cores)
    run_forward(emb, idx, off, B)
    emb.backward(torch.as_tensor(go, device=DEV), lr=lr)
    assert emb.check() == 0
    sv = emb.state_views() or [None] * cfg.num_tables
    for t, cv in enumerate(emb.core_views()):
        for k in range(3):
            ref_p, ref_s = Oracle.update(opt, lr, cores[t][k], g[t][k], None)
            assert_update_close(cv[k].cpu().numpy(), ref_p, cores[t][k], g[t][k], ga[t][k], lr, opt,
                                got_s=None if sv[t] is None else sv[t][k].cpu().numpy(), ref_s=ref_s,
                                s_old=np.zeros_like(cores[t][k]), what=f"c4 fused {opt} t{t} C{k+1}")


@pytest.mark.parametrize("rank", [32, 64, 128])
def test_c5_full_size_sampled(rank):
    """Multi-hot c5 shape (8 x 40 M rows, N = 128, L = 20) at B = 16384 per GPU (a quarter of the
    global 65 536) in the bench launch configuration.  Plan bit-exact vs numpy on the whole batch;
    64 sampled bags vs the oracle; core gradients of sampled slices of table 0: for core k and a
    sample S_k of digits (the most frequent one plus two random ones), the oracle runs on the
    sub-batch of the positions whose k-th digit lies in S_k -- a slice's gradient depends only on
    those positions, so the comparison is exact, hot slices included."""
    cfg = W.config("c5", rank)
    B = 16384
    idx, off = W.make_batch(cfg, seed=5, batch=B)
    cores = W.make_cores(cfg, seed=5)
    go = W.make_grad_out(cfg, B, seed=5)
    emb = gpu_emb(cfg, B, len(idx))
    emb.load_cores(cores)
    out = run_forward(emb, idx, off, B).cpu().numpy()
    assert emb.check() == 0
    _check_plan_full(emb, cfg, idx, off, B)
    T = cfg.num_tables
    orc = Oracle.from_config(cfg)
    rng = np.random.default_rng(0)
    bs = np.sort(rng.choice(B, size=64, replace=False))
    keep = np.zeros(len(idx), bool)
    for t in range(T):
        for b in bs:
            keep[off[t * B + b]:off[t * B + b + 1]] = True
    bag_sel = np.zeros(T * B, bool)
    for t in range(T):
        bag_sel[t * B + bs] = True
    sub_off = np.concatenate([[0], np.cumsum(np.diff(off)[bag_sel.reshape(T, B).ravel()])]).astype(np.int64)
    sidx = idx[keep]
    ref = orc.forward(cores, sidx, sub_off, len(bs))
    ref_abs = orc.forward(cores, sidx, sub_off, len(bs), absolute=True)
    assert_companion(out[bs], ref, ref_abs, 1e-5, "sampled forward")
    emb.backward(torch.as_tensor(go, device=DEV))
    assert emb.check() == 0
    grads = emb.grad_views()[0]
    tab = np.repeat(np.arange(T * B), np.diff(off)) // B
    on0 = tab == 0
    dig = np.stack(np.unravel_index(np.where(on0, idx, 0), tuple(cfg.row_factors[0])))
    for k in range(3):
        present, cnt = np.unique(dig[k][on0], return_counts=True)
        sample = {int(present[np.argmax(cnt)])}
        sample |= set(int(x) for x in rng.choice(present, size=min(2, len(present)), replace=False))
        sample = np.array(sorted(sample))
        sel = on0 & np.isin(dig[k], sample)
        soff = _sub_batch(off, sel)
        gk = orc.backward(cores, idx[sel], soff, B, go)[0][k]
        gka = orc.backward(cores, idx[sel], soff, B, go, absolute=True)[0][k]
        mine = grads[k].cpu().numpy()
        assert_companion(mine[sample], gk[sample], gka[sample], 1e-4, f"c5 r{rank} dC{k+1} slices {sample}")


def test_fused_update_sgd_and_adagrad():
    cfg = W.small_config([500, 300], [(8, 8, 8), (7, 7, 7)], (2, 2, 4), 16, 64, 2, 1.05)
    idx, off = W.make_batch(cfg, seed=2)
    cores = W.make_cores(cfg, seed=2)
    go = W.make_grad_out(cfg, cfg.batch, seed=2)
    orc = Oracle.from_config(cfg)
    g = orc.backward(cores, idx, off, cfg.batch, go)
    ga = orc.backward(cores, idx, off, cfg.batch, go, absolute=True)
    lr = 0.05
    for opt in ("sgd", "adagrad"):
        for fused in (True, False):
            emb = gpu_emb(cfg, cfg.batch, len(idx), optimizer=opt, fused_update=fused)
            emb.load_cores(cores)
            run_forward(emb, idx, off, cfg.batch)
            emb.backward(torch.as_tensor(go, device=DEV), lr=lr)
            if not fused:
                emb.update(lr)
            else:
                with pytest.raises(tt.TTEmbError):
                    emb.update(lr)
            torch.cuda.synchronize()
            for t, (cv, sv) in enumerate(zip(emb.core_views(),
                                             emb.state_views() or [None] * cfg.num_tables)):
                for k in range(3):
                    ref_p, ref_s = Oracle.update(opt, lr, cores[t][k], g[t][k], None)
                    assert_update_close(cv[k].cpu().numpy(), ref_p, cores[t][k], g[t][k], ga[t][k], lr,
                                        opt, got_s=None if sv is None else sv[k].cpu().numpy(),
                                        ref_s=ref_s, s_old=np.zeros_like(cores[t][k]),
                                        what=f"{opt} fused={fused} t{t} C{k+1}")


def test_two_steps_match_oracle_trajectory():
    """Two fused SGD steps: the second step's gradients use the updated cores."""
    cfg = W.small_config([1000], [(10, 10, 10)], (2, 2, 4), 8, 64, 1, 1.05)
    cores = W.make_cores(cfg, seed=4)
    emb = gpu_emb(cfg, cfg.batch, cfg.batch, fused_update=True)
    emb.load_cores(cores)
    orc = Oracle.from_config(cfg)
    lr = 0.1
    ref_cores = [tuple(x.copy() for x in c) for c in cores]
    for step in range(2):
        idx, off = W.make_batch(cfg, step=step, seed=4)
        go = W.make_grad_out(cfg, cfg.batch, step=step, seed=4)
        run_forward(emb, idx, off, cfg.batch)
        emb.backward(torch.as_tensor(go, device=DEV), lr=lr)
        g = orc.backward(ref_cores, idx, off, cfg.batch, go)
        ref_cores = [tuple(Oracle.update("sgd", lr, c[k], g[t][k])[0] for k in range(3))
                     for t, c in enumerate(ref_cores)]
    for cv, rc in zip(emb.core_views(), ref_cores):
        for k in range(3):
            np.testing.assert_allclose(cv[k].cpu().numpy(), rc[k], rtol=1e-4, atol=1e-5)


def test_int32_indices_and_host_api():
    cfg = W.config("c2")
    B = 512
    idx, off = W.make_batch(cfg, seed=9, batch=B)
    cores = W.make_cores(cfg, seed=9)
    go = W.make_grad_out(cfg, B, seed=9)
    e64 = gpu_emb(cfg, B, len(idx))
    e64.load_cores(cores)
    o64 = run_forward(e64, idx, off, B)
    e64.backward(torch.as_tensor(go, device=DEV))
    e32 = gpu_emb(cfg, B, len(idx), index_bits=32)
    e32.load_cores(cores)
    o32 = run_forward(e32, idx, off, B, index_bits=32)
    e32.backward(torch.as_tensor(go, device=DEV))
    torch.testing.assert_close(o32, o64, rtol=0, atol=0)
    eh = gpu_emb(cfg, B, len(idx))
    eh.load_cores(cores)
    hi = torch.as_tensor(idx).pin_memory()
    ho = torch.as_tensor(off).pin_memory()
    hout = torch.empty(B, cfg.num_tables, cfg.dim).pin_memory()
    eh.forward_host(hi, ho, B, hout)
    eh.backward_host(torch.as_tensor(go).pin_memory())
    torch.cuda.synchronize()
    torch.testing.assert_close(hout, o64.cpu(), rtol=0, atol=0)
    # the aggregated row gradients and dC1 are summed with vector reductions in arrival order
    # (R19 / Q19): runs agree up to fp32 reassociation
    for a, b in zip(eh.grad_views(), e64.grad_views()):
        for k in range(3):
            torch.testing.assert_close(a[k], b[k], rtol=1e-5, atol=1e-5 * float(b[k].abs().max()))


def test_deterministic_forward_and_plan():
    cfg = W.config("c3")
    B = 2048
    idx, off = W.make_batch(cfg, seed=1, batch=B)
    cores = W.make_cores(cfg, seed=1)
    emb = gpu_emb(cfg, B, len(idx))
    emb.load_cores(cores)
    o1 = run_forward(emb, idx, off, B).clone()
    p1 = emb.plan()
    o2 = run_forward(emb, idx, off, B)
    p2 = emb.plan()
    torch.testing.assert_close(o1, o2, rtol=0, atol=0)
    for k in ("ukey", "inverse", "grp_pfx", "row_seg"):
        assert torch.equal(p1[k], p2[k])


def test_pdl_launch_order_does_not_change_results(tmp_path):
    """The main chain is launched with programmatic dependent launch; with it switched off
    (TTEMB_NO_PDL=1, read once per process, hence the subprocesses) the forward output -- which
    has no atomics, so it is deterministic -- is bitwise equal (c4 shapes, B = 1024)."""
    import os
    import subprocess
    import sys
    code = (
        "import sys, numpy as np, torch\n"
        "sys.path.insert(0, {root!r})\n"
        "import paper_conf_sc_wangwfmmd22_b200 as tt\n"
        "from synth import workload as W\n"
        "cfg = W.config('c4'); B = 1024\n"
        "idx, off = W.make_batch(cfg, seed=3, batch=B)\n"
        "emb = tt.TTEmbeddingBag(cfg.table_rows, cfg.row_factors, cfg.col_factors, cfg.rank, B, len(idx))\n"
        "emb.load_cores(W.make_cores(cfg, seed=3))\n"
        "d = torch.device('cuda', 0)\n"
        "out = emb.forward(torch.as_tensor(idx, device=d), torch.as_tensor(off, device=d), B)\n"
        "np.save({out!r}, out.cpu().numpy())\n"
    )
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    res = []
    for flag in ("0", "1"):
        f = str(tmp_path / f"out{flag}.npy")
        env = dict(os.environ, TTEMB_NO_PDL=flag)
        r = subprocess.run([sys.executable, "-c", code.format(root=root, out=f)], env=env, cwd=root,
                           capture_output=True, text=True, timeout=300)
        assert r.returncode == 0, r.stderr[-2000:]
        res.append(np.load(f))
    np.testing.assert_array_equal(res[0], res[1])


def test_edge_cases_empty_and_range_errors():
    cfg = W.small_config([100, 50], [(5, 5, 4), (4, 4, 4)], (2, 2, 2), 4, 8, 1)
    cores = W.make_cores(cfg, seed=0)
    emb = gpu_emb(cfg, 8, 64)
    emb.load_cores(cores)
    # all bags empty
    off = np.zeros(2 * 8 + 1, np.int64)
    out = run_forward(emb, np.zeros(0, np.int64), off, 8)
    emb.backward(torch.zeros(8, 2, 8, device=DEV))
    assert emb.check() == 0
    assert float(out.abs().sum()) == 0.0
    assert emb.counts()["U"] == 0
    for v in emb.grad_views():
        for x in v:
            assert float(x.abs().sum()) == 0.0
    # batch 0
    out = run_forward(emb, np.zeros(0, np.int64), np.zeros(1, np.int64), 0)
    assert out.numel() == 0 and emb.check() == 0
    # id out of range (>= M, including padding ids < m1 m2 m3) -> INDEX_RANGE
    idx = np.array([5, 100, 3, 1, 0, 2, 4, 6, 7, 8, 9, 10, 11, 12, 13, 14], np.int64)
    off = np.arange(17, dtype=np.int64)
    run_forward(emb, idx, off, 8)
    assert emb.check() == L.TTEMB_ERR_INDEX_RANGE
    idx[1] = -1
    run_forward(emb, idx, off, 8)
    assert emb.check() == L.TTEMB_ERR_INDEX_RANGE
    # malformed offsets -> INVALID_ARG (deferred)
    bad = off.copy()
    bad[3], bad[4] = bad[4], bad[3]
    idx[1] = 1
    run_forward(emb, idx, bad, 8)
    assert emb.check() == L.TTEMB_ERR_INVALID_ARG
    # capacity and state errors are synchronous
    with pytest.raises(tt.TTEmbError):
        run_forward(emb, np.zeros(65, np.int64), np.concatenate([np.zeros(16, np.int64), [65]]), 8)
    fresh = gpu_emb(cfg, 8, 64)
    with pytest.raises(tt.TTEmbError):
        fresh.backward(torch.zeros(0, 2, 8, device=DEV))
    # exactly one backward per forward (a second one would double the plan's accumulators)
    idx = np.arange(16, dtype=np.int64) % 7
    run_forward(emb, idx, np.arange(17, dtype=np.int64), 8)
    emb.backward(torch.zeros(8, 2, 8, device=DEV))
    with pytest.raises(tt.TTEmbError):
        emb.backward(torch.zeros(8, 2, 8, device=DEV))


ABLATIONS = [dict(prefix_reuse=False), dict(aggregation=False), dict(prefix_reuse=False, aggregation=False)]


@pytest.mark.parametrize("abl", ABLATIONS, ids=["no-reuse", "no-agg", "no-reuse-no-agg"])
@pytest.mark.parametrize("case", ["dup-heavy", "tc-multitile", "c4-b1024", "c4-b1024-fp32"])
def test_ablation_switches(case, abl):
    """TTEMB_NO_PREFIX_REUSE / TTEMB_NO_AGGREGATION (the paper's Fig. 14/17/18 toggles)
    change only the amount of work: outputs and core gradients still match the oracle, and the
    plan counts become U = nnz (no dedup / aggregation) and P = U (no prefix reuse)."""
    kw = {}
    if case.startswith("c4"):
        cfg, mode, B = W.config("c4"), None, 1024
        kw["fp32_cores"] = case.endswith("fp32")
    else:
        cfg, mode = {c[0]: (c[1], c[2]) for c in small_cases()}[case]
        B = None
    idx, off, B = make_inputs(cfg, mode, seed=5, batch=B)
    cores = W.make_cores(cfg, seed=5)
    go = W.make_grad_out(cfg, B, seed=5)
    emb = gpu_emb(cfg, B, len(idx), **kw, **abl)
    emb.load_cores(cores)
    out = run_forward(emb, idx, off, B)
    emb.backward(torch.as_tensor(go, device=DEV))
    assert emb.check() == 0
    orc = Oracle.from_config(cfg)
    ref_plan = orc.plan(idx, off, B)
    cnt = emb.counts()
    U = len(idx) if abl.get("aggregation") is False else ref_plan["U"]
    assert cnt["U"] == U
    if abl.get("prefix_reuse") is False:
        assert cnt["P"] == U
    elif abl.get("aggregation") is False:
        assert cnt["P"] == ref_plan["P"]   # duplicates share their prefix run
    assert_companion(out.cpu().numpy(), orc.forward(cores, idx, off, B),
                     orc.forward(cores, idx, off, B, absolute=True), 1e-5, "forward")
    g = orc.backward(cores, idx, off, B, go)
    ga = orc.backward(cores, idx, off, B, go, absolute=True)
    for t, mine in enumerate(emb.grad_views()):
        for k in range(3):
            assert_companion(mine[k].cpu().numpy(), g[t][k], ga[t][k], 1e-4, f"dC{k+1} t{t}")


@pytest.mark.parametrize("case", ["multi-var-L", "tc-multitile", "c4-b1024"])
def test_runtime_bijection(case):
    """ttemb_set_bijection: the CUDA path looks up New_Batch = {index(i_j)}; outputs and
    gradients match the oracle applied to the mapped ids; the plan is the plan of the mapped ids."""
    from paper_conf_sc_wangwfmmd22_b200 import reorder
    if case.startswith("c4"):
        cfg, mode, B = W.config("c4").replace(id_map="perm"), None, 1024
    else:
        cfg, mode = {c[0]: (c[1], c[2]) for c in small_cases()}[case]
        B = None
    idx, off, B = make_inputs(cfg, mode, seed=9, batch=B)
    hist = [W.make_batch(cfg, step=s, seed=9, batch=B) + (B,) for s in range(1, 4)]
    bij = reorder.frequency_bijection(cfg.table_rows, hist)
    maps = reorder.split_bijection(bij, cfg.table_rows)
    cores = W.make_cores(cfg, seed=9)
    go = W.make_grad_out(cfg, B, seed=9)
    emb = gpu_emb(cfg, B, len(idx))
    emb.load_cores(cores)
    emb.set_bijection(torch.as_tensor(bij.view(np.int32), device=DEV))
    out = run_forward(emb, idx, off, B)
    emb.backward(torch.as_tensor(go, device=DEV))
    assert emb.check() == 0
    orc = Oracle.from_config(cfg)
    mid = orc.apply_bijection(maps, idx, off, B)
    check_plan(emb, orc, mid, off, B)
    assert_companion(out.cpu().numpy(), orc.forward(cores, mid, off, B),
                     orc.forward(cores, mid, off, B, absolute=True), 1e-5, "forward")
    g = orc.backward(cores, mid, off, B, go)
    ga = orc.backward(cores, mid, off, B, go, absolute=True)
    for t, mine in enumerate(emb.grad_views()):
        for k in range(3):
            assert_companion(mine[k].cpu().numpy(), g[t][k], ga[t][k], 1e-4, f"dC{k+1} t{t}")
    # switching it off restores the raw-id lookup
    emb.set_bijection(None)
    out2 = run_forward(emb, idx, off, B)
    emb.backward(torch.as_tensor(go, device=DEV))
    assert emb.check() == 0
    check_plan(emb, orc, idx, off, B)


def test_bijection_out_of_range_is_reported():
    cfg = W.config("c1")
    idx, off = W.make_batch(cfg, seed=1)
    emb = gpu_emb(cfg, cfg.batch, len(idx))
    bad = np.arange(cfg.table_rows[0], dtype=np.int32)
    bad[int(idx[0])] = cfg.table_rows[0]            # maps a used id outside [0, M)
    emb.set_bijection(torch.as_tensor(bad, device=DEV))
    run_forward(emb, idx, off, cfg.batch)
    assert emb.check() == L.TTEMB_ERR_INDEX_RANGE


@pytest.mark.parametrize("mode,weighted", [("mean", False), ("sum", True)], ids=["mean", "weighted"])
@pytest.mark.parametrize("case", ["multi-var-L", "tc-n1-2", "c4-b1024-var", "c4-b1000-one"])
def test_mean_and_weighted_bags(case, mode, weighted):
    """nn.EmbeddingBag mode="mean" (TTEMB_MEAN_POOLING) and per-sample weights
    (ttemb_forward_weighted) vs the oracle's definition (P:48 / P:306 drop-in); variable bag
    lengths with empty bags; the backward differentiates the weighted bags.  The one-hot case
    (B = 1000, ragged against every tile) runs the output-ordered one-hot pooling kernel."""
    if case.startswith("c4"):
        cfg, B = W.config("c4"), int(case.split("-")[1][1:])
        mode_in = "var" if case.endswith("var") else None
    else:
        cfg, mode_in = {c[0]: (c[1], c[2]) for c in small_cases()}[case]
        mode_in, B = "var", None
    idx, off, B = make_inputs(cfg, mode_in, seed=13, batch=B)
    psw = np.random.default_rng(13).uniform(-2, 2, size=len(idx)).astype(np.float32) if weighted else None
    cores = W.make_cores(cfg, seed=13)
    go = W.make_grad_out(cfg, B, seed=13)
    emb = gpu_emb(cfg, B, len(idx), mode=mode)
    emb.load_cores(cores)
    it = torch.as_tensor(idx.astype(np.int64), device=DEV)
    out = emb.forward(it, torch.as_tensor(off, device=DEV), B,
                      per_sample_weights=torch.as_tensor(psw, device=DEV) if weighted else None)
    emb.backward(torch.as_tensor(go, device=DEV))
    assert emb.check() == 0
    orc = Oracle.from_config(cfg)
    kw = dict(per_sample_weights=psw, mode=mode)
    assert_companion(out.cpu().numpy(), orc.forward(cores, idx, off, B, **kw),
                     orc.forward(cores, idx, off, B, absolute=True, **kw), 1e-5, "forward")
    g = orc.backward(cores, idx, off, B, go, **kw)
    ga = orc.backward(cores, idx, off, B, go, absolute=True, **kw)
    for t, mine in enumerate(emb.grad_views()):
        for k in range(3):
            assert_companion(mine[k].cpu().numpy(), g[t][k], ga[t][k], 1e-4, f"dC{k+1} t{t}")


def test_weights_with_mean_rejected_by_the_abi():
    cfg = W.config("c1")
    idx, off = W.make_batch(cfg, seed=1)
    emb = gpu_emb(cfg, cfg.batch, len(idx), mode="mean")
    with pytest.raises(tt.TTEmbError):
        emb.forward(torch.as_tensor(idx, device=DEV), torch.as_tensor(off, device=DEV), cfg.batch,
                    per_sample_weights=torch.ones(len(idx), device=DEV))


HYBRID = {
    "small-ffma": lambda: W.hybrid(W.small_config([37, 300, 5, 1000], [(3, 4, 4), (7, 7, 7), (1, 2, 3), (10, 10, 10)],
                                                  (2, 3, 2), 4, 24, 1, 1.05), threshold=100),
    "tc-r64": lambda: W.hybrid(W.small_config([20000, 300, 5000, 40], [(28, 28, 26), (7, 7, 7), (18, 18, 16), (4, 4, 3)],
                                              (4, 4, 4), 64, 96, 1, 1.05), threshold=1000),
    "c4-hybrid-b1024": lambda: W.hybrid(W.config("c4")),
}


@pytest.mark.parametrize("case", list(HYBRID))
def test_hybrid_placement(case):
    """Hybrid placement (TTEMB table.dense): small tables are plain EmbeddingBag tables in the
    same call.  Plan (TT-first keys, dense rows without prefix), forward, dW / dC_k vs the oracle;
    variable bag lengths."""
    cfg = HYBRID[case]()
    B = 1024 if case.startswith("c4") else None
    idx, off, B = make_inputs(cfg, "var", seed=17, batch=B)
    cores = W.make_cores(cfg, seed=17)
    go = W.make_grad_out(cfg, B, seed=17)
    emb = gpu_emb(cfg, B, len(idx))
    emb.load_cores(cores)
    out = run_forward(emb, idx, off, B)
    emb.backward(torch.as_tensor(go, device=DEV))
    assert emb.check() == 0
    orc = Oracle.from_config(cfg)
    check_plan(emb, orc, idx, off, B)
    assert_companion(out.cpu().numpy(), orc.forward(cores, idx, off, B),
                     orc.forward(cores, idx, off, B, absolute=True), 1e-5, "forward")
    g = orc.backward(cores, idx, off, B, go)
    ga = orc.backward(cores, idx, off, B, go, absolute=True)
    for t, mine in enumerate(emb.grad_views()):
        for k in range(3):
            if g[t][k].size:
                assert_companion(mine[k].cpu().numpy(), g[t][k], ga[t][k], 1e-4, f"dC{k+1} t{t}")


@pytest.mark.parametrize("opt", ["sgd", "adagrad"])
def test_hybrid_fused_update(opt):
    """Dense rows are updated in place by the backward (fused, one replica) exactly like the
    unfused backward + ttemb_update; TT cores as before."""
    cfg = HYBRID["tc-r64"]()
    idx, off = W.make_batch(cfg, seed=19)
    B = cfg.batch
    cores = W.make_cores(cfg, seed=19)
    go = W.make_grad_out(cfg, B, seed=19)
    orc = Oracle.from_config(cfg)
    g = orc.backward(cores, idx, off, B, go)
    ga = orc.backward(cores, idx, off, B, go, absolute=True)
    lr = 0.05
    for fused in (True, False):
        emb = gpu_emb(cfg, B, len(idx), optimizer=opt, fused_update=fused)
        emb.load_cores(cores)
        run_forward(emb, idx, off, B)
        emb.backward(torch.as_tensor(go, device=DEV), lr=lr)
        if not fused:
            emb.update(lr)
        torch.cuda.synchronize()
        for t, (cv, sv) in enumerate(zip(emb.core_views(), emb.state_views() or [None] * cfg.num_tables)):
            for k in range(3):
                if not cores[t][k].size:
                    continue
                ref_p, ref_s = Oracle.update(opt, lr, cores[t][k], g[t][k], None)
                assert_update_close(cv[k].cpu().numpy(), ref_p, cores[t][k], g[t][k], ga[t][k], lr,
                                    opt, got_s=None if sv is None else sv[k].cpu().numpy(),
                                    ref_s=ref_s, s_old=np.zeros_like(cores[t][k]),
                                    what=f"{opt} fused={fused} t{t} C{k+1}")


@pytest.mark.parametrize("case", ["c1", "tc-r64"])
def test_pipelined_plan_on_side_stream(case):
    """ttemb_plan_batch / ttemb_forward_planned with two handles on the same cores (the bench's
    cross-step pipelining): batch s+1's index stage runs on a side stream during batch s's
    forward + fused SGD backward; three steps follow the oracle's trajectory and the plans match."""
    if case == "c1":
        cfg = W.small_config([1000], [(10, 10, 10)], (2, 2, 4), 8, 64, 1, 1.05)
    else:
        cfg = W.small_config([20000, 300], [(28, 28, 26), (7, 7, 7)], (4, 4, 4), 64, 96, 1, 1.05)
    B = cfg.batch
    cores = W.make_cores(cfg, seed=6)
    emb = gpu_emb(cfg, B, B * cfg.num_tables, fused_update=True)
    emb.load_cores(cores)
    embs = [emb, emb.sibling()]
    orc = Oracle.from_config(cfg)
    lr = 0.1
    batches = [W.make_batch(cfg, step=s, seed=6) for s in range(4)]
    gos = [W.make_grad_out(cfg, B, step=s, seed=6) for s in range(4)]
    dev = [(torch.as_tensor(i, device=DEV), torch.as_tensor(o, device=DEV)) for i, o in batches]
    side = torch.cuda.Stream()
    cur = torch.cuda.current_stream()
    embs[0].plan_batch(dev[0][0], dev[0][1], B)
    ref = [tuple(x.copy() for x in c) for c in cores]
    outs = []
    for s in range(3):
        h, nh = embs[s % 2], embs[(s + 1) % 2]
        go_ = cur.record_event()
        out = h.forward_planned()
        side.wait_event(go_)
        nh.plan_batch(dev[s + 1][0], dev[s + 1][1], B, stream=side)
        pl = side.record_event()
        h.backward(torch.as_tensor(gos[s], device=DEV), lr=lr)
        cur.wait_event(pl)
        outs.append(out.cpu().numpy())
        idx, off = batches[s]
        # step 0 reads the initial cores: the north-star forward tolerance; later steps read cores
        # that already carry one fp32 update rounding per step
        assert_companion(outs[-1], orc.forward(ref, idx, off, B), orc.forward(ref, idx, off, B, absolute=True),
                         1e-5 if s == 0 else 1e-4, f"forward step {s}")
        g = orc.backward(ref, idx, off, B, gos[s])
        ref = [tuple(Oracle.update("sgd", lr, c[k], g[t][k])[0] for k in range(3)) for t, c in enumerate(ref)]
    torch.cuda.synchronize()
    for cv, rc in zip(emb.core_views(), ref):
        for k in range(3):
            np.testing.assert_allclose(cv[k].cpu().numpy(), rc[k], rtol=1e-4, atol=1e-5)
    with pytest.raises(tt.TTEmbError):            # forward_planned needs a fresh plan
        embs[0].forward_planned()


@pytest.mark.parametrize("rank", [16, 128])
@pytest.mark.parametrize("opt", ["sgd", "adagrad"])
def test_ffma_split_groups_fused_and_unfused(opt, rank):
    """FFMA path (TTEMB_FP32_CORES) with Zipf-hot i2-groups of more than kGroupChunk (128)
    prefixes: a group is split over several CTAs (asserted through the plan's split-group
    counter), its dC2 partials meet by reductions and (fused) a separate pass updates the slice.
    Gradients (unfused) and updated cores (fused) vs the oracle; a second fused step starts from
    cleared split-group accumulators."""
    cfg = W.small_config([200000], [(2000, 10, 10)], (2, 2, 4), rank, 2048, 4, 0.9)
    idx, off = W.make_batch(cfg, seed=23)
    B = cfg.batch
    cores = W.make_cores(cfg, seed=23)
    go = W.make_grad_out(cfg, B, seed=23)
    orc = Oracle.from_config(cfg)
    plan = orc.plan(idx, off, B)
    sizes = np.diff(plan["grp_off"])
    assert sizes.max() > 128, sizes.max()          # the case must contain split groups
    g = orc.backward(cores, idx, off, B, go)
    ga = orc.backward(cores, idx, off, B, go, absolute=True)
    lr = 0.05
    for fused in (False, True):
        emb = gpu_emb(cfg, B, len(idx), optimizer=opt, fused_update=fused, fp32_cores=True)
        emb.load_cores(cores)
        run_forward(emb, idx, off, B)
        assert emb.all_counts()["nsplit"] > 0      # the split-group machinery ran
        emb.backward(torch.as_tensor(go, device=DEV), lr=lr)
        if not fused:
            for k in range(3):
                assert_companion(emb.grad_views()[0][k].cpu().numpy(), g[0][k], ga[0][k], 1e-4, f"dC{k+1}")
            emb.update(lr)
        torch.cuda.synchronize()
        sv = emb.state_views()
        for k in range(3):
            ref_p, ref_s = Oracle.update(opt, lr, cores[0][k], g[0][k], None)
            assert_update_close(emb.core_views()[0][k].cpu().numpy(), ref_p, cores[0][k], g[0][k], ga[0][k], lr,
                                opt, got_s=None if sv is None else sv[0][k].cpu().numpy(), ref_s=ref_s,
                                s_old=np.zeros_like(cores[0][k]), what=f"{opt} fused={fused} C{k+1}")
        if fused:
            # second step from the updated cores: split-group accumulators must have been cleared
            cur = [tuple(v.cpu().numpy().copy() for v in emb.core_views()[0])]
            cur_s = None if sv is None else [tuple(v.cpu().numpy().copy() for v in sv[0])]
            run_forward(emb, idx, off, B)
            emb.backward(torch.as_tensor(go, device=DEV), lr=lr)
            assert emb.check() == 0
            g2 = orc.backward(cur, idx, off, B, go)
            g2a = orc.backward(cur, idx, off, B, go, absolute=True)
            torch.cuda.synchronize()
            for k in range(3):
                ref_p, ref_s = Oracle.update(opt, lr, cur[0][k], g2[0][k], None if cur_s is None else cur_s[0][k])
                assert_update_close(emb.core_views()[0][k].cpu().numpy(), ref_p, cur[0][k], g2[0][k], g2a[0][k],
                                    lr, opt, got_s=None if sv is None else emb.state_views()[0][k].cpu().numpy(),
                                    ref_s=ref_s, s_old=None if cur_s is None else cur_s[0][k],
                                    what=f"{opt} step 2 C{k+1}")


@pytest.mark.parametrize("rank,storage", [(40, 64), (20, 32)])
def test_rank_padding_storage_is_exact(rank, storage):
    """16 <= R < 32 and 32 < R < 64 run on the tcgen05 path with cores stored zero-padded to rank
    32 / 64 (ttemb_config.rank doc, R28): the padding stays exactly zero through fused
    SGD and Adagrad steps, and the results match the oracle at the configured rank."""
    cfg = W.small_config([20000, 300], [(28, 28, 26), (7, 7, 7)], (4, 4, 4), rank, 96, 2, 1.05)
    idx, off = W.make_batch(cfg, seed=29)
    B = cfg.batch
    cores = W.make_cores(cfg, seed=29)
    go = W.make_grad_out(cfg, B, seed=29)
    orc = Oracle.from_config(cfg)
    for opt in ("sgd", "adagrad"):
        emb = gpu_emb(cfg, B, len(idx), optimizer=opt, fused_update=True)
        assert emb.layout[0][1][1][1] == storage         # storage rank of C2
        emb.load_cores(cores)
        out = run_forward(emb, idx, off, B)
        assert_companion(out.cpu().numpy(), orc.forward(cores, idx, off, B),
                         orc.forward(cores, idx, off, B, absolute=True), 1e-5, "forward")
        for _ in range(2):
            run_forward(emb, idx, off, B)
            emb.backward(torch.as_tensor(go, device=DEV), lr=0.05)
        torch.cuda.synchronize()
        R = cfg.rank
        for t in range(cfg.num_tables):
            full = []
            for k in range(3):
                o, shp = emb.layout[t][k]
                shp = shp if k == 1 else shp[:3]
                full.append(emb.cores[o:o + int(np.prod(shp))].view(*shp))
            assert torch.count_nonzero(full[0][:, :, R:]) == 0
            assert torch.count_nonzero(full[1][:, R:]) == 0 and torch.count_nonzero(full[1][..., R:]) == 0
            assert torch.count_nonzero(full[2][:, R:]) == 0
            assert torch.count_nonzero(full[1][:, :R, :, :R]) > 0


@pytest.mark.parametrize("opt", ["sgd", "adagrad"])
def test_checkpoint_resume_round_trip(opt):
    """state_dict -> torch.save -> torch.load -> load_state_dict into a fresh instance restores
    cores and optimizer state bit for bit; the restored instance's forward is bitwise the
    original's and the next training step agrees with the uninterrupted one (to fp32 reduction
    order: dC1 / dC3 sums use reductions); a mismatched config is rejected."""
    import io
    cfg = W.small_config([5000, 70000], [(17, 17, 18), (41, 41, 42)], (4, 4, 4), 64, 512, 1, 1.05)
    kw = dict(fused_update=True, optimizer=opt)
    nnz = cfg.batch * cfg.num_tables
    a = gpu_emb(cfg, cfg.batch, nnz, **kw)
    a.load_cores(W.make_cores(cfg, seed=21))
    for step in range(2):
        idx, off = W.make_batch(cfg, step=step, seed=21)
        run_forward(a, idx, off, cfg.batch)
        a.backward(torch.as_tensor(W.make_grad_out(cfg, cfg.batch, step=step, seed=21), device=DEV), lr=0.05)
    buf = io.BytesIO()
    torch.save(a.state_dict(), buf)
    buf.seek(0)
    b = gpu_emb(cfg, cfg.batch, nnz, **kw)
    b.load_state_dict(torch.load(buf))
    assert torch.equal(a.cores, b.cores)
    if opt == "adagrad":
        assert torch.equal(a.state, b.state)
    idx, off = W.make_batch(cfg, step=2, seed=21)
    oa = run_forward(a, idx, off, cfg.batch).clone()
    ob = run_forward(b, idx, off, cfg.batch).clone()
    assert torch.equal(oa, ob)
    go = torch.as_tensor(W.make_grad_out(cfg, cfg.batch, step=2, seed=21), device=DEV)
    a.backward(go, lr=0.05)
    b.backward(go, lr=0.05)
    torch.cuda.synchronize()
    ca, cb = a.cores.cpu().numpy(), b.cores.cpu().numpy()
    assert np.linalg.norm(cb - ca) <= 1e-6 * np.linalg.norm(ca)
    other = gpu_emb(cfg.replace(rank=32), cfg.batch, nnz, **kw)
    with pytest.raises(ValueError):
        other.load_state_dict(a.state_dict())


def test_host_step_pipeline_matches_device_steps():
    """HostStepPipeline (pinned host inputs / outputs, copies overlapped with compute) computes
    the same outputs and the same trained cores as device-resident steps."""
    cfg = W.small_config([5000, 70000], [(17, 17, 18), (41, 41, 42)], (4, 4, 4), 64, 512, 1, 1.05)
    cores = W.make_cores(cfg, seed=22)
    steps = [(W.make_batch(cfg, step=k, seed=22), W.make_grad_out(cfg, cfg.batch, step=k, seed=22)) for k in range(4)]
    nnz = cfg.batch * cfg.num_tables
    a = gpu_emb(cfg, cfg.batch, nnz, fused_update=True)
    a.load_cores(cores)
    ref = []
    for (idx, off), go in steps:
        ref.append(run_forward(a, idx, off, cfg.batch).cpu().numpy())
        a.backward(torch.as_tensor(go, device=DEV), lr=0.05)
    b = gpu_emb(cfg, cfg.batch, nnz, fused_update=True)
    b.load_cores(cores)
    pipe = tt.HostStepPipeline(b, nnz, cfg.batch, depth=2)
    outs = [torch.empty(cfg.batch, cfg.num_tables, cfg.dim).pin_memory() for _ in steps]
    hin = [(torch.as_tensor(i).pin_memory(), torch.as_tensor(o).pin_memory(), torch.as_tensor(g).pin_memory())
           for (i, o), g in steps]
    ks = [pipe.step(hi, ho, hg, outs[k], lr=0.05) for k, (hi, ho, hg) in enumerate(hin)]
    pipe.wait(ks[-1])
    torch.cuda.synchronize()
    # step 0 runs on identical cores: bitwise; later steps differ by the reduction order of the
    # earlier updates: normwise fp32-level agreement
    np.testing.assert_array_equal(outs[0].numpy(), ref[0])
    for k in range(1, len(steps)):
        assert np.linalg.norm(outs[k].numpy() - ref[k]) <= 1e-5 * np.linalg.norm(ref[k]), k
    ca, cb = a.cores.cpu().numpy(), b.cores.cpu().numpy()
    assert np.linalg.norm(cb - ca) <= 1e-6 * np.linalg.norm(ca)
