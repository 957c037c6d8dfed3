"""Beyond-memory streaming (mp_compute_stream): the same
P and I as the in-memory path, bit for bit, for every precision, self- and AB-join, warp-tile and
block-cooperative kernels, with the device holding only one row window and one column window of
the per-position arrays at a time.  The in-memory path itself is oracle-checked in
test_gpu_parity.py; the planted motif is also checked against the oracle here.
"""
import os

import numpy as np
import pytest

from paper_conf_ipps_juryl022_b200 import datagen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def ctx():
    """Re-seed intervals of 256 / 256 / 64 / 64 rows (FP64 / FP32 / FP16 / Mixed): the tile
    height follows them at these sizes, so one row chunk is a few hundred rows in every mode."""
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_juryl022_b200 import mstamp
    c = mstamp.Context(0, reseed_h=[256, 256, 64, 64])
    yield c
    c.close()


class _Geo:
    """Force a fine chunk geometry through the library's testing knobs."""

    def __init__(self, rows, diags):
        self.v = {"MP_STREAM_ROWS": str(rows), "MP_STREAM_DIAGS": str(diags)}

    def __enter__(self):
        os.environ.update(self.v)

    def __exit__(self, *a):
        for k in self.v:
            os.environ.pop(k, None)


def _same(ctx, T, m, prec, e, Tr=None, rows=1, diags=1, budget=1 << 30):
    P0, I0 = ctx.compute(T, m, prec, e, Tr=Tr)
    with _Geo(rows, diags):
        P1, I1 = ctx.compute_stream(T, m, prec, e, Tr=Tr, device_bytes=budget)
    R, Wb, peak, nl = ctx.last_stream_info()
    assert np.array_equal(P0, P1, equal_nan=True), (prec, float(np.nanmax(np.abs(P0 - P1))))
    assert np.array_equal(I0, I1), (prec, int((I0 != I1).sum()))
    return R, Wb, peak, nl


@pytest.mark.parametrize("prec", ["fp64", "fp32", "mixed", "fp16ck", "fp16c", "fp16"])
@pytest.mark.parametrize("shape", [(4, 3000, 32, 8, 201), (16, 2100, 48, 12, 202), (64, 1800, 24, 6, 203)])
def test_stream_self_bit_identical(ctx, prec, shape):
    """Self-join, many row chunks x diagonal bands (rows = one tile height, a few blocks per
    band): bit-identical to mp_compute; d = 4 / 16 warp-tile kernels, d = 64 block kernels."""
    d, n, m, e, seed = shape
    T = datagen.random_walk(d, n, m, seed) if prec in ("fp64", "fp32") else datagen.bounded_patterns(d, n, m, seed)
    R, Wb, peak, nl = _same(ctx, T, m, prec, e, rows=1, diags=150)
    print(prec, shape, "R", R, "Wb", Wb, "launches", nl, "peak MiB", peak / 2**20)
    assert R < n and nl > 4


@pytest.mark.parametrize("prec", ["fp64", "fp32", "mixed", "fp16"])
@pytest.mark.parametrize("shape", [(5, 2500, 24, 211), (70, 1200, 16, 212)])
def test_stream_ab_bit_identical(ctx, prec, shape):
    """AB-join (diagonals in (-n, n), query keys only), chunked: bit-identical to mp_compute."""
    d, n, m, seed = shape
    if prec in ("fp64", "fp32"):
        Tq, Tr = datagen.random_walk_ab(d, n, m, seed)
    else:
        Tq, Tr = datagen.bounded_patterns(d, n, m, seed), datagen.bounded_patterns(d, n, m, seed + 1000)
    R, Wb, peak, nl = _same(ctx, Tq, m, prec, -1, Tr=Tr, rows=1, diags=200)
    print(prec, shape, "R", R, "Wb", Wb, "launches", nl)
    assert R < n and nl > 4


def test_stream_c1_matches_oracle_motif(ctx, oracle_mod):
    """C1 streamed in FP64 equals the in-memory result and recovers the oracle's planted motif."""
    cfg = datagen.make("C1")
    T, m, e, n = cfg["T"], cfg["m"], cfg["exclusion"], cfg["n"]
    _same(ctx, T, m, "fp64", e, rows=1, diags=500)
    with _Geo(1, 500):
        P, I = ctx.compute_stream(T, m, "fp64", e)
    a, b = datagen.motif_positions(n, m)
    Po, Io, _ = oracle_mod.mstamp(T, m, e, rows=np.array([a, b]))
    assert np.array_equal(I[:, [a, b]], Io)
    assert np.allclose(P[:, [a, b]], Po, rtol=1e-9, atol=1e-6)


def test_stream_large_exclusion_rows_without_cells(ctx):
    """Rows no band reaches (exclusion >= n - 1 - i) keep P = +inf, I = -1 (reading G3)."""
    d, n, m = 3, 1500, 16
    T = datagen.random_walk(d, n, m, 221)
    e = n - 200
    _same(ctx, T, m, "fp32", e, rows=1, diags=64)
    with _Geo(1, 64):
        P, I = ctx.compute_stream(T, m, "fp32", e)
    assert np.all(np.isinf(P[:, 200:n - 200])) and np.all(I[:, 200:n - 200] == -1)


def test_stream_auto_geometry_budget(ctx):
    """Automatic geometry from a device budget: chunked, peak mapped memory within the budget,
    bit-identical to the in-memory path (d = 64: the TMA block kernel)."""
    from paper_conf_ipps_juryl022_b200 import mstamp
    d, n, m, e = 64, 24576, 64, 16
    T = datagen.random_walk(d, n, m, 231)
    budget = 160 << 20
    R_plan, Wb_plan = mstamp.plan_stream(d, n, m, "fp32", e, True, budget)
    assert R_plan < n
    P0, I0 = ctx.compute(T, m, "fp32", e)
    P1, I1 = ctx.compute_stream(T, m, "fp32", e, device_bytes=budget)
    R, Wb, peak, nl = ctx.last_stream_info()
    print("R", R, "Wb", Wb, "peak MiB", peak / 2**20, "launches", nl)
    assert (R, Wb) == (R_plan, Wb_plan)
    assert peak <= budget
    assert np.array_equal(P0, P1) and np.array_equal(I0, I1)
    ms, nl2 = ctx.last_timing()
    assert ms > 0 and nl2 == nl


def test_stream_budget_too_small(ctx):
    from paper_conf_ipps_juryl022_b200 import mstamp
    T = datagen.random_walk(64, 20000, 64, 241)
    with pytest.raises(mstamp.MPError) as ei:
        ctx.compute_stream(T, 64, "fp32", 16, device_bytes=8 << 20)
    assert ei.value.status == 2   # MP_ERR_NOMEM
    # the context stays usable
    P, I = ctx.compute(T[:, :3000], 64, "fp32", 16)
    assert np.all(np.isfinite(P))


def test_stream_rejects_non_finite(ctx):
    from paper_conf_ipps_juryl022_b200 import mstamp
    T = datagen.random_walk(4, 2000, 32, 251)
    T[2, 1500] = np.nan
    with _Geo(1, 100):
        with pytest.raises(mstamp.MPError) as ei:
            ctx.compute_stream(T, 32, "fp32", 8)
    assert ei.value.status == 1
