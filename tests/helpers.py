"""Shared test helpers: tolerance metric and GPU runners."""
from __future__ import annotations

import numpy as np


def assert_companion(got, ref, ref_abs, tol, what=""):
    """|got - ref| <= tol * ref_abs elementwise (forward-error bound of a sum of
    products; ref_abs = the same computation on |inputs|), plus the normwise
    ||got - ref|| <= tol * ||ref_abs||.  Exact zeros must stay exact."""
    got = np.asarray(got, dtype=np.float64).reshape(np.shape(ref))
    err = np.abs(got - ref)
    bound = tol * np.asarray(ref_abs) + 1e-30
    bad = err > bound
    if bad.any():
        i = np.flatnonzero(bad.ravel())[:5]
        raise AssertionError(
            f"{what}: {bad.sum()} / {bad.size} elements exceed tol {tol}: "
            f"got {got.ravel()[i]}, ref {np.asarray(ref).ravel()[i]}, bound {bound.ravel()[i]}")
    n_ref = np.linalg.norm(np.asarray(ref_abs).ravel())
    assert np.linalg.norm(err.ravel()) <= tol * n_ref + 1e-30, what


def assert_update_close(got_p, ref_p, p_old, g_ref, g_abs, lr, opt, tol=1e-4, got_s=None,
                        ref_s=None, s_old=None, eps=1e-10, what=""):
    """Updated cores (and Adagrad state) against the oracle update of the oracle
    gradient.  The bound propagates the gradient tolerance through the update
    rule plus fp32 rounding of the result."""
    got_p = np.asarray(got_p, np.float64).ravel()
    ref_p = np.asarray(ref_p, np.float64).ravel()
    p_old = np.asarray(p_old, np.float64).ravel()
    g = np.asarray(g_ref, np.float64).ravel()
    ga = np.asarray(g_abs, np.float64).ravel()
    dg = tol * ga                                   # admissible gradient error
    ulp = 4 * np.finfo(np.float32).eps * (np.abs(p_old) + np.abs(ref_p))
    if opt == "sgd":
        bound = lr * dg + ulp
    else:
        s0 = np.asarray(s_old, np.float64).ravel()
        s = s0 + g * g
        # d/dg [g / sqrt(s0 + g^2)] = s0 / (s0+g^2)^1.5 <= 1/sqrt(s0+g^2); ill-conditioned
        # where |g| ~ dg and s0 ~ 0: allow the full step there.
        # An untouched element (g_abs = 0, so dg = 0) must stay put up to rounding: its bound is
        # the ulp term alone (without the mask, 0 * inf = NaN would make it unfailable).
        touched = dg > 0
        with np.errstate(divide="ignore", invalid="ignore", over="ignore"):
            sens = np.where(s > (10 * dg) ** 2, 1.0 / np.sqrt(np.maximum(s, 1e-300)), np.inf)
            step = np.where(touched, np.minimum(lr * dg * sens * 2, 2 * lr), 0.0)
        bound = step + ulp
        assert not np.isnan(bound).any(), what
        if got_s is not None:
            gs = np.asarray(got_s, np.float64).ravel()
            rs = np.asarray(ref_s, np.float64).ravel()
            sb = 2 * np.abs(g) * dg + dg * dg + 4 * np.finfo(np.float32).eps * rs
            bad = np.abs(gs - rs) > sb + 1e-30
            assert not bad.any(), f"{what} state: {bad.sum()} bad"
    err = np.abs(got_p - ref_p)
    bad = err > bound
    if bad.any():
        i = np.flatnonzero(bad)[:5]
        raise AssertionError(f"{what}: {bad.sum()} / {bad.size} updated params off: got {got_p[i]}, "
                             f"ref {ref_p[i]}, bound {bound[i]}")


def plan_key(cfg, idx, off, B):
    """Group-major plan key of every position (R29): kbase_t + (i2 m1 + i1) m3 + i3,
    digits (i1, i2, i3) of Eq. 3 via numpy.unravel_index per table."""
    T = cfg.num_tables
    mf = np.array(cfg.row_factors, np.int64)
    kbase = np.concatenate([[0], np.cumsum(mf.prod(axis=1))[:-1]]).astype(np.int64)
    bag = np.repeat(np.arange(T * B), np.diff(off))
    tab = bag // B
    key = np.empty(len(idx), np.int64)
    for t in range(T):
        sel = tab == t
        d1, d2, d3 = np.unravel_index(np.asarray(idx)[sel], tuple(mf[t]))
        key[sel] = kbase[t] + (d2 * mf[t, 0] + d1) * mf[t, 2] + d3
    return key
