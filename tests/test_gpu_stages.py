"""Per-stage unit tests: one stage of the hot path at a time, on the device, through
the C ABI's stage self-test entry points (include/mp.h), with the fused kernels' own device code.

* the d-way sort + inclusive scan (Eq. 2) of every FP32 kernel variant, on
  values built to break a sorting network: exact ties, +inf, denormals, zeros, already sorted and
  reversed rows; checked against numpy's sort and a float64 cumulative sum;
* the precalculation (reading G7; FP32 mode: FP64 rounded once, R1') against
  the oracle's window statistics and df / dg formed from them in numpy.
"""
import math

import numpy as np
import pytest

from paper_conf_ipps_juryl022_b200 import datagen

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def ctx():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_juryl022_b200 import mstamp
    c = mstamp.Context(0)
    yield c
    c.close()


def _hard_rows(d, count, seed):
    rng = np.random.default_rng(seed)
    X = rng.uniform(0, 40, size=(count, d)).astype(np.float32)
    X[0] = 3.5                                            # all ties
    X[1] = np.arange(d, dtype=np.float32)                 # sorted
    X[2] = np.arange(d, dtype=np.float32)[::-1]           # reversed
    if d & (d - 1) == 0:                                  # +inf (no padded dims to sort after it)
        X[3, ::2] = np.inf
    else:                                                 # the largest distance, 2 sqrt(m) at m = 512
        X[3, ::2] = np.float32(2 * math.sqrt(512))
    X[4] = np.float32(1e-40)                              # denormals (FTZ-free compares)
    X[4, d // 2:] = 0.0
    X[5] = np.round(X[5])                                 # many ties among few values
    X[6, : d // 3] = 0.0                                  # exact zeros (planted-motif distances)
    return X


@pytest.mark.parametrize("d", [1, 3, 4, 8, 13, 16, 17, 32, 33, 64, 100, 128, 256, 512])
def test_sort_scan_stage(ctx, d):
    X = _hard_rows(d, 300, d)
    got = ctx.selftest_sort_scan(X)
    want = np.cumsum(np.sort(X.astype(np.float64), axis=1), axis=1)
    fin = np.isfinite(want)
    assert np.array_equal(fin, np.isfinite(got)), "inf pattern differs"
    # the kernels sum in a different (pairwise / two-chain) order than numpy: FP32 rounding only
    tol = 4 * d * 2.0 ** -24 * np.abs(want) + 1e-44
    assert np.all(np.abs(got[fin] - want[fin]) <= tol[fin])
    # the sort itself is exact: the first prefix sum is the minimum, bit for bit
    assert np.array_equal(got[:, 0], np.sort(X, axis=1)[:, 0])


@pytest.mark.parametrize("prec", ["fp64", "fp32"])
@pytest.mark.parametrize("d,n,m", [(3, 500, 16), (16, 300, 64), (70, 200, 32)])
def test_precompute_stage(ctx, oracle_mod, prec, d, n, m):
    T = datagen.random_walk(d, n, m, 91)
    T[0, 40:40 + 2 * m] = 2.5                              # flat windows: a = 0 (reading G4)
    df, dg, a = ctx.selftest_precompute(T, m, prec)
    mu, nrm = oracle_mod.window_stats(T, m)                # (d, n) each, two-pass long double
    L = n + m - 1
    df_w = np.zeros((n, d))
    dg_w = np.zeros((n, d))
    df_w[1:] = ((T[:, m:L] - T[:, : n - 1]) / 2.0).T        # reading G7
    dg_w[1:] = ((T[:, m:L] - mu[:, 1:]) + (T[:, : n - 1] - mu[:, :-1])).T
    a_w = np.where(nrm > 0, math.sqrt(2 * m) / np.where(nrm > 0, nrm, 1.0), 0.0).T
    scale = np.abs(T).max() + 1.0
    rtol = 1e-12 if prec == "fp64" else 2.0 ** -23
    assert np.allclose(df, df_w, rtol=rtol, atol=rtol * scale)
    assert np.allclose(dg, dg_w, rtol=rtol, atol=rtol * scale)
    flat = a_w == 0
    assert np.all(a[flat] == 0)
    assert np.allclose(a[~flat], a_w[~flat], rtol=1e-12 if prec == "fp64" else 2.0 ** -23, atol=0)
