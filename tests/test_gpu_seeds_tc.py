"""Tensor-core seeds (mp_config.seed_mode = MP_SEEDS_TC).

The seed GEMM alone (mp_selftest_seeds) against the definition in FP64 (PAPER.md:L586-588:
direct centred dot products at the re-seed rows), with the rigorous error bound of FP16 operands
and FP32 accumulation; then the whole Mixed / FP16CK path with tensor-core seeds against the
oracle within the half modes' stated bound, band partials merging bit-identically, and the
accuracy next to the CUDA-core seeds.
"""
import math

import numpy as np
import pytest

from paper_conf_ipps_juryl022_b200 import datagen

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

U16 = 2.0 ** -11   # unit roundoff of FP16 (round to nearest)
U32 = 2.0 ** -24


@pytest.fixture(scope="module")
def ctx_tc():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_juryl022_b200 import mstamp
    c = mstamp.Context(0, seed_mode="tc")
    yield c
    c.close()


@pytest.fixture(scope="module")
def ctx_direct():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    from paper_conf_ipps_juryl022_b200 import mstamp
    c = mstamp.Context(0)
    yield c
    c.close()


def _windows(x, m, starts):
    W = np.lib.stride_tricks.sliding_window_view(x, m)[starts]
    return W - W.mean(axis=1, keepdims=True)


@pytest.mark.parametrize("case", [  # (d, n, m, H, ab, seed)
    (4, 3000, 100, 256, False, 301),    # m not a multiple of 16 (zero-padded K), ragged last tiles
    (3, 2000, 512, 128, False, 302),    # K = 512: eight operand chunks through the double buffer
    (5, 1500, 64, 64, True, 303),       # AB-join: rows from T, columns from Tr
])
def test_seed_gemm_vs_definition(ctx_tc, case):
    """Every seed of the table against the FP64 definition: |S - S_64| <= u16 |S_64| (final
    rounding to half) + (2 u16 + m u32) sum_t |a_t b_t| (FP16 operands, FP32 accumulation)."""
    d, n, m, H, ab, seed = case
    if ab:
        T, Tr = datagen.random_walk_ab(d, n, m, seed)
    else:
        T, Tr = datagen.random_walk(d, n, m, seed), None
    nr = (n + H - 1) // H
    tab, sc = ctx_tc.selftest_seeds(T, m, "mixed", H=H, rows=(0, nr), Tr=Tr)
    sq = sc[:d]
    sr = sc[d:] if ab else sq
    worst = 0.0
    for k in range(d):
        A = _windows(sq[k] * T[k], m, np.arange(nr) * H)
        B = _windows(sr[k] * (Tr if ab else T)[k], m, np.arange(n))
        ref = A @ B.T
        mag = np.abs(A) @ np.abs(B).T
        tol = U16 * np.abs(ref) + (2 * U16 + m * U32) * mag + 1e-30
        err = np.abs(tab[:, k, :] - ref)
        assert np.all(err <= tol), (k, float((err / tol).max()))
        worst = max(worst, float((err / tol).max()))
    print(case, "max err / bound", worst)


@pytest.mark.parametrize("prec", ["mixed", "fp16ck"])
@pytest.mark.parametrize("shape", [(64, 2500, 32, 8, 311), (100, 900, 64, 16, 312), (64, 1200, 48, -1, 313)])
def test_tc_seeds_path_vs_oracle(ctx_tc, oracle_mod, prec, shape):
    """The whole path with tensor-core seeds (block half kernels, d >= 64), self- and AB-join,
    against the oracle within the half modes' stated element-wise bound (test_gpu_parity.HALF_BOUND)."""
    from test_gpu_parity import _assert_half_bound
    d, n, m, e, seed = shape
    T = datagen.bounded_patterns(d, n, m, seed)
    Tr = datagen.bounded_patterns(d, n, m, seed + 1000) if e < 0 else None
    P, I, _ = oracle_mod.mstamp(T, m, None if e < 0 else e, Tr=Tr)
    Pg, Ig = ctx_tc.compute(T, m, prec, e, Tr=Tr)
    assert np.all(np.isfinite(Pg)) and np.all((Ig >= 0) & (Ig < n))
    print(prec, shape, "element-wise", _assert_half_bound(P, Pg, m, prec))


@pytest.mark.parametrize("prec", ["mixed"])
def test_tc_seeds_bands_merge_bit_identically(ctx_tc, prec):
    """Band partials (each with its own row-chunked seed tables) merge to the single band bit for bit."""
    from paper_conf_ipps_juryl022_b200 import mstamp
    d, n, m = 64, 1800, 32
    T = torch.from_numpy(datagen.bounded_patterns(d, n, m, 321)).cuda()
    kw = mstamp.key_words(d, n, prec)
    full = torch.empty(kw, dtype=torch.int64, device="cuda")
    ctx_tc.partial_device(T, m, full, 0, 1, prec, 8)
    parts = []
    for r in range(3):
        k = torch.empty(kw, dtype=torch.int64, device="cuda")
        ctx_tc.partial_device(T, m, k, r, 3, prec, 8)
        parts.append(k)
    merged = torch.stack(parts).min(dim=0).values
    torch.cuda.synchronize()
    assert torch.equal(merged, full)


def test_tc_seeds_accuracy_vs_direct(ctx_tc, ctx_direct):
    """Random walk with a planted motif (X64-like shape): tensor-core and CUDA-core seeds both
    inside the stated Mixed bound vs the FP64 path over the full grid, the motif recovered, and the
    tensor-core seeds' error of the same order as the direct seeds' (FP16 operands vs FP32)."""
    from test_gpu_parity import _assert_half_bound
    d, n, m, e = 64, 8192, 256, 64
    T = datagen.random_walk(d, n, m, 331)
    P64, _ = ctx_direct.compute(T, m, "fp64", e)
    Pd, _ = ctx_direct.compute(T, m, "mixed", e)
    Pt, It = ctx_tc.compute(T, m, "mixed", e)
    bd = _assert_half_bound(P64, Pd, m, "mixed")
    bt = _assert_half_bound(P64, Pt, m, "mixed")
    print("direct (max, p99.9)", bd, "tc", bt)
    assert bt[1] <= 2.0 * bd[1] + 1e-3
    a, b = datagen.motif_positions(n, m)
    assert abs(int(It[0, a]) - b) <= m // 16
