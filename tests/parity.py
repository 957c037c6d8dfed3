"""Acceptance rules of GPU results vs the FP64 oracle.

P:  |P_gpu - P_or| <= rtol * P_or                      (general)
    |P_gpu - P_or| <= rtol * P_or + sqrt(2 m rho_tol)   (near-exact: P_or < 0.05 sqrt(2m))
I:  I_gpu == I_or where the oracle's runner-up gap P2 - P exceeds tol(P); elsewhere any
    I_gpu whose own oracle value D''_k(i, I_gpu) <= P_or + tol(P) is accepted.
"""
import math

import numpy as np

TOL = {"fp64": (1e-9, 1e-12), "fp32": (1e-4, 1e-5)}


def tol_of(P_or, m, prec):
    rtol, rho_tol = TOL[prec]
    near = P_or < 0.05 * math.sqrt(2 * m)
    return rtol * np.abs(P_or) + np.where(near, math.sqrt(2 * m * rho_tol), 0.0)


def check(oracle, T, m, P_or, I_or, P2_or, P_gpu, I_gpu, prec, rows=None, Tr=None):
    """Assert parity; returns a stats dict.  rows: query rows of the oracle arrays (sampled)."""
    d = P_or.shape[0]
    Pg = P_gpu if rows is None else P_gpu[:, rows]
    Ig = I_gpu if rows is None else I_gpu[:, rows]
    rowid = np.arange(P_or.shape[1]) if rows is None else np.asarray(rows)
    fin = np.isfinite(P_or)
    assert np.array_equal(fin, np.isfinite(Pg)), "finite pattern differs"
    assert np.all(Ig[~fin] == -1) and np.all(I_or[~fin] == -1)
    tol = tol_of(np.where(fin, P_or, 0.0), m, prec)
    err = np.abs(np.where(fin, Pg - P_or, 0.0))
    bad = err > tol
    assert not bad.any(), f"P parity: {bad.sum()} entries, worst {err[bad].max() if bad.any() else 0}"
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
