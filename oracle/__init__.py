"""FP64 CPU oracle for mSTAMP -- TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s cpu_baseline /
``--impl reference`` leg may import this package.  It never imports the CUDA
product package and the product package never imports it.

The arithmetic lives in plain C (``mstamp_oracle.c``; see its header for the
definition and the PAPER.md passages it follows).  This module only builds
(gcc) and marshals arguments via ctypes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "mstamp_oracle.c")
_LIB = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (IEEE double; no -ffast-math, no FMA contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        subprocess.check_call(
            ["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-shared", "-fPIC",
             "-pthread", "-o", _LIB, _SRC, "-lm"])
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        i64, p = ctypes.c_int64, ctypes.c_void_p
        lib.oracle_window_stats.argtypes = [p, i64, i64, i64, p, p]
        lib.oracle_cell.argtypes = [p, p, i64, i64, i64, i64, i64, p]
        lib.oracle_mstamp.argtypes = [p, p, i64, i64, i64, i64, p, i64, ctypes.c_int, p, p, p]
        lib.oracle_cells.argtypes = [p, p, i64, i64, i64, p, p, i64, p]
        lib.oracle_mstamp_band.argtypes = [p, p, i64, i64, i64, i64, p, i64, i64, i64, ctypes.c_int, p, p, p]
        for f in (lib.oracle_window_stats, lib.oracle_cell, lib.oracle_mstamp, lib.oracle_cells,
                  lib.oracle_mstamp_band):
            f.restype = ctypes.c_int
        _lib = lib
    return _lib


def _ptr(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


def _series(T):
    T = np.ascontiguousarray(T, dtype=np.float64)
    if T.ndim == 1:
        T = T[None, :]
    return T


def window_stats(T, m):
    """Per-(k,i) window mean and norm ||x - mu|| (two-pass).  Returns (mu, norm), each d x n."""
    T = _series(T)
    d, L = T.shape
    n = L - m + 1
    mu = np.empty((d, n))
    nrm = np.empty((d, n))
    rc = _load().oracle_window_stats(_ptr(T), d, n, m, _ptr(mu), _ptr(nrm))
    assert rc == 0
    return mu, nrm


def cell(T, m, i, j, Tr=None):
    """D''_k(i, j) for all k (length-d vector) of one cell."""
    T = _series(T)
    d, L = T.shape
    n = L - m + 1
    Tr_ = None if Tr is None else _series(Tr)
    out = np.empty(d)
    rc = _load().oracle_cell(_ptr(T), _ptr(Tr_), d, n, m, int(i), int(j), _ptr(out))
    assert rc == 0
    return out


def cells(T, m, ii, jj, Tr=None):
    """D''_k(ii[c], jj[c]) for all k: array (count, d)."""
    T = _series(T)
    d, L = T.shape
    n = L - m + 1
    Tr_ = None if Tr is None else _series(Tr)
    ii = np.ascontiguousarray(ii, dtype=np.int64)
    jj = np.ascontiguousarray(jj, dtype=np.int64)
    out = np.empty((len(ii), d))
    rc = _load().oracle_cells(_ptr(T), _ptr(Tr_), d, n, m, _ptr(ii), _ptr(jj), len(ii), _ptr(out))
    assert rc == 0
    return out


def mstamp(T, m, exclusion=None, Tr=None, rows=None, nthreads=None):
    """Matrix profile by definition.

    T: (d, L) float64 query series (L = n + m - 1).  Tr: reference series for an
    AB-join, or None for a self-join.  exclusion: self-join skips |i-j| <= e;
    None or negative -> ceil(m/4) (reading G1).  rows: optional query rows to
    evaluate (sampled parity); default all n.
    Returns (P, I, P2), each (d, nrows); P2 is the runner-up value.
    """
    T = _series(T)
    d, L = T.shape
    n = L - m + 1
    if exclusion is None or exclusion < 0:
        exclusion = -(-m // 4)
    Tr_ = None if Tr is None else _series(Tr)
    if Tr_ is not None:
        assert Tr_.shape == T.shape, "AB-join needs equal lengths (reading G22)"
    if rows is None:
        r = None
        nrows = n
    else:
        r = np.ascontiguousarray(rows, dtype=np.int64)
        nrows = len(r)
    P = np.empty((d, nrows))
    P2 = np.empty((d, nrows))
    I = np.empty((d, nrows), dtype=np.int64)
    nt = nthreads or os.cpu_count() or 1
    rc = _load().oracle_mstamp(_ptr(T), _ptr(Tr_), d, n, m, int(exclusion), _ptr(r), nrows,
                               int(nt), _ptr(P), _ptr(I), _ptr(P2))
    assert rc == 0
    return P, I, P2


def mstamp_band(T, m, rows, dlo, dhi, exclusion=None, Tr=None, nthreads=None):
    """Partial profile of one diagonal band for query rows: min / argmin /
    runner-up over the cells with delta = j - i (AB-join) or |j - i| (self-join) in
    [dlo, dhi), self-join exclusion as in mstamp().  Returns (P, I, P2), each (d, len(rows))."""
    T = _series(T)
    d, L = T.shape
    n = L - m + 1
    if exclusion is None or exclusion < 0:
        exclusion = -(-m // 4)
    Tr_ = None if Tr is None else _series(Tr)
    r = np.ascontiguousarray(rows, dtype=np.int64)
    nrows = len(r)
    P = np.empty((d, nrows))
    P2 = np.empty((d, nrows))
    I = np.empty((d, nrows), dtype=np.int64)
    nt = nthreads or os.cpu_count() or 1
    rc = _load().oracle_mstamp_band(_ptr(T), _ptr(Tr_), d, n, m, int(exclusion), _ptr(r), nrows,
                                    int(dlo), int(dhi), int(nt), _ptr(P), _ptr(I), _ptr(P2))
    assert rc == 0
    return P, I, P2
