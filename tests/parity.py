"""Acceptance rules of GPU results vs the FP64 oracle.

P:  |P_gpu - P_or| <= rtol * P_or                      (general)
    |P_gpu - P_or| <= rtol * P_or + sqrt(2 m rho_tol)   (near-exact: P_or < 0.05 sqrt(2m))
I:  I_gpu == I_or where the oracle's runner-up gap P2 - P exceeds tol(P); elsewhere any
    I_gpu whose own oracle value D''_k(i, I_gpu) <= P_or + tol(P) is accepted.
"""
import math
import os

import numpy as np

TOL = {"fp64": (1e-9, 1e-12), "fp32": (1e-4, 1e-5)}


def tol_of(P_or, m, prec, P0_row=None):
    """Tolerance per (k, i).  A distance component near D = 0 carries an absolute error up to
    sqrt(2 m rho_tol) (D = sqrt(2m(1-rho)) turns a rho error into sqrt of it), and it enters
    every k-dim mean that includes it.  Such a component exists in row i only if the row's
    best single-dimension match is near-exact, i.e. P[0][i] < 0.05 sqrt(2m); for those rows
    the floor applies to all k."""
    rtol, rho_tol = TOL[prec]
    thr = 0.05 * math.sqrt(2 * m)
    near = P_or < thr
    if P0_row is not None:
        near = near | (P0_row[None, :] < thr)
    return rtol * np.abs(P_or) + np.where(near, math.sqrt(2 * m * rho_tol), 0.0)


def kappa(T, m):
    """Per-window conditioning of FP32 storage: max_k max|x| / ||x - mu|| over the window's dims.
    Rounding the input to FP32 perturbs a z-normalised window by <= m * 2^-24 * kappa (DESIGN.md
    "Tolerances"); flat or offset-dominated windows (large kappa) are the paper's ill-conditioned
    case."""
    T = np.atleast_2d(T)
    w = np.lib.stride_tricks.sliding_window_view(T, m, axis=1)
    amax = np.abs(w).max(axis=2)
    nrm = np.sqrt(((w - w.mean(axis=2, keepdims=True)) ** 2).sum(axis=2))
    with np.errstate(divide="ignore"):
        k = np.where(nrm > 0, amax / np.where(nrm > 0, nrm, 1), np.inf)
    return k.max(axis=0)


def check(oracle, T, m, P_or, I_or, P2_or, P_gpu, I_gpu, prec, rows=None, Tr=None, cond=False):
    """Assert parity; returns a stats dict.  rows: query rows of the oracle arrays (sampled).
    cond=True (FP32 on generic, possibly ill-conditioned inputs) adds the input-rounding term
    8 m 2^-24 (kappa_i + kappa_j) to the tolerance; BASELINE configs are checked without it."""
    d = P_or.shape[0]
    Pg = P_gpu if rows is None else P_gpu[:, rows]
    Ig = I_gpu if rows is None else I_gpu[:, rows]
    rowid = np.arange(P_or.shape[1]) if rows is None else np.asarray(rows)
    fin = np.isfinite(P_or)
    assert np.array_equal(fin, np.isfinite(Pg)), "finite pattern differs"
    assert np.all(Ig[~fin] == -1) and np.all(I_or[~fin] == -1)
    tol = tol_of(np.where(fin, P_or, 0.0), m, prec, P0_row=np.where(fin[0], P_or[0], np.inf))
    if cond and prec == "fp32" and not os.environ.get("MP_PARITY_NO_COND"):
        kq = kappa(T, m)
        kr = kq if Tr is None else kappa(Tr, m)
        kj = kr[np.clip(I_or, 0, len(kr) - 1)]
        tol = tol + np.where(fin, 8 * m * 2.0 ** -24 * (kq[rowid][None, :] + kj), 0.0)
    err = np.abs(np.where(fin, Pg - P_or, 0.0))
    bad = err > tol
    if bad.any():
        ks, cs = np.nonzero(bad)
        det = [(int(k), int(rowid[c]), float(P_or[k, c]), float(Pg[k, c]), float(P_or[0, c])) for k, c in
               list(zip(ks, cs))[:8]]
        raise AssertionError(f"P parity: {bad.sum()} entries (k, i, P_or, P_gpu, P_or[0,i]): {det}")
    with np.errstate(invalid="ignore"):
        gap = np.where(fin, P2_or - P_or, np.inf)
    strict = fin & (gap > tol)
    exact = strict & (Ig == I_or)
    n_strict_fail = int((strict & (Ig != I_or)).sum())
    assert n_strict_fail == 0, f"I parity: {n_strict_fail} strict mismatches"
    amb = fin & ~strict & (Ig != I_or)
    n_amb = int(amb.sum())
    if n_amb:
        ks, cs = np.nonzero(amb)
        vals = oracle.cells(T, m, rowid[cs], Ig[ks, cs], Tr=Tr)
        v = vals[np.arange(len(ks)), ks]
        ok = v <= P_or[ks, cs] + tol[ks, cs]
        assert ok.all(), f"ambiguous index not within tolerance: {(~ok).sum()}"
    rel = np.where(fin & (P_or > 0), err / np.where(P_or > 0, P_or, 1), 0.0)
    return dict(max_rel=float(rel.max()), exact_idx=int(exact.sum()), ambiguous_ok=n_amb,
                near=int((fin & (P_or < 0.05 * math.sqrt(2 * m))).sum()), count=int(fin.sum()))
