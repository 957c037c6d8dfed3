"""Pins of the FP64 CPU oracle against things other than itself (CPU only).

Each test names the PAPER.md passage or the mathematical fact it rests on.
A plausible mistake in the oracle (dropped centring, sigma vs sample sigma,
wrong sort direction, sum instead of mean, wrong index orientation, lost
exclusion zone, lost tie rule) fails at least one of them.
"""
import math
import os

import numpy as np
import pytest

import brute
from paper_conf_ipps_juryl022_b200 import datagen

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _near_tol(P_ref, m, rtol=1e-12, rho_tol=1e-12):
    # |dP| <= rtol * P + sqrt(2 m rho_tol) for near-exact matches
    near = P_ref < 0.05 * math.sqrt(2 * m)
    return rtol * P_ref + np.where(near, math.sqrt(2 * m * rho_tol), 0.0)


def _check_index(P_or, I_or, P2_or, I_b, P_b, tol):
    # index must agree where the runner-up gap exceeds the tolerance
    with np.errstate(invalid="ignore"):
        gap = P2_or - P_or
    strict = np.nan_to_num(gap, nan=0.0) > tol
    assert np.array_equal(I_or[strict], I_b[strict])


# ---------------------------------------------------------------- Eq. (1) vs definition
@pytest.mark.parametrize("d,n,m,e,seed", [(1, 60, 8, 2, 1), (3, 90, 16, 4, 2), (5, 185, 16, 4, 3),
                                          (4, 120, 7, 0, 4), (2, 64, 32, 40, 5)])
def test_oracle_vs_znormalised_bruteforce(oracle_mod, d, n, m, e, seed):
    """Eq. (1) sqrt(2m(1-rho)) == Euclidean distance of z-normalised windows."""
    T = datagen.random_walk(d, n, m, seed, motif=False)
    P, I, P2 = oracle_mod.mstamp(T, m, e)
    Pb, Ib, P2b = brute.mstamp(T, m, e)
    tol = _near_tol(Pb, m, rtol=1e-11)
    fin = np.isfinite(Pb)
    assert np.array_equal(fin, np.isfinite(P))
    assert np.all(np.abs(P[fin] - Pb[fin]) <= tol[fin] + 1e-13)
    _check_index(P, I, P2, Ib, Pb, 1e-9)
    # the runner-up (the value the index rule of tests/parity.py rests on) against the brute force
    fin2 = np.isfinite(P2b)
    assert np.array_equal(fin2, np.isfinite(P2))
    assert np.all(np.abs(P2[fin2] - P2b[fin2]) <= _near_tol(P2b, m, rtol=1e-11)[fin2] + 1e-13)


def test_oracle_ab_join_vs_bruteforce(oracle_mod):
    Tq, Tr = datagen.random_walk_ab(3, 80, 12, 7, motif=False)
    P, I, P2 = oracle_mod.mstamp(Tq, 12, Tr=Tr)
    Pb, Ib, P2b = brute.mstamp(Tq, 12, 0, Tr=Tr)
    assert np.allclose(P, Pb, rtol=1e-11, atol=1e-12)
    assert np.allclose(P2, P2b, rtol=1e-11, atol=1e-12)
    _check_index(P, I, P2, Ib, Pb, 1e-9)


def _plant_copies(T, m, src, dsts):
    """Exact copies of window src at each window start in dsts, in every dimension: the copied
    windows are bit-identical, so every query ties exactly between them (and src)."""
    T = T.copy()
    for x in dsts:
        T[:, x:x + m] = T[:, src:src + m]
    return T


@pytest.mark.parametrize("ab", [False, True])
def test_runner_up_with_exact_ties(oracle_mod, ab):
    """Runner-up P2 (the oracle's best2, Eq. (3) L538-549 + reading G2) against the brute
    force on inputs with planted exact ties: where the argmin ties with a bit-identical copy, the
    oracle must report P2 == P (a tie is not a strict gap) and the lowest tied index (G2);
    elsewhere P2 equals the brute-force second-best value."""
    d, n, m = 3, 70, 8
    if ab:
        Tq, Tr = datagen.random_walk_ab(d, n, m, 41, motif=False)
        Tr = _plant_copies(Tr, m, 10, [30, 55])
        P, I, P2 = oracle_mod.mstamp(Tq, m, Tr=Tr)
        Pb, Ib, P2b = brute.mstamp(Tq, m, 0, Tr=Tr)
    else:
        Tq, Tr = _plant_copies(datagen.random_walk(d, n, m, 41, motif=False), m, 5, [30, 52]), None
        P, I, P2 = oracle_mod.mstamp(Tq, m, 2)
        Pb, Ib, P2b = brute.mstamp(Tq, m, 2)
    tol = _near_tol(Pb, m, rtol=1e-11) + 1e-13
    assert np.all(np.abs(P - Pb) <= tol)
    assert np.all(np.abs(P2 - P2b) <= _near_tol(P2b, m, rtol=1e-11) + 1e-13)
    copies = {10, 30, 55} if ab else {5, 30, 52}
    tied = np.isin(I, list(copies))
    assert tied.sum() > 0
    # an exact tie between bit-identical windows: runner-up equals the best, index is the lowest copy
    for k, i in zip(*np.nonzero(tied)):
        others = [j for j in copies if j != I[k, i] and (ab or abs(j - i) > 2)]
        if others:
            assert P2[k, i] == P[k, i], (k, i)
            assert I[k, i] == min([I[k, i]] + others), (k, i)
    # away from ties, the strict gap is positive and the index agrees with the brute force
    _check_index(P, I, P2, Ib, Pb, 1e-9)
    assert np.mean((P2 - P) > 1e-9) > 0.5


def test_cell_matches_direct_definition(oracle_mod):
    T = datagen.random_walk(6, 50, 10, 11, motif=False)
    D = brute.dist_cube(T, 10)
    for (i, j) in [(0, 30), (7, 41), (40, 3), (12, 12)]:
        s = np.cumsum(np.sort(D[:, i, j])) / np.arange(1, 7)
        # i == j: D ~ sqrt(2m * eps) rounding residue on both sides (near-exact floor)
        atol = 1e-6 if i == j else 1e-12
        assert np.allclose(oracle_mod.cell(T, 10, i, j), s, rtol=1e-12, atol=atol)


# ---------------------------------------------------------------- golden, hand-derived
def _read_golden(name):
    rows, dims, meta = [], [], {}
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.strip()
            if not line or line.startswith("#"):
                continue
            tok = line.split()
            if tok[0].startswith("dim"):
                dims.append([float(v) for v in tok[1:]])
            elif tok[0] in ("m", "exclusion"):
                meta[tok[0]] = int(tok[1])
            else:
                i, k, p, idx = int(tok[0]), int(tok[1]), float(tok[2]), tok[3]
                rows.append((i, k, p, {int(v) for v in idx.split(",")}))
    return np.array(dims), meta, rows


def test_golden_m2_hand_derived(oracle_mod):
    """tests/golden/m2_selfjoin.txt: closed-form m=2 profile (Eqs. 1-3, readings G1, G2, G4)."""
    T, meta, rows = _read_golden("m2_selfjoin.txt")
    P, I, _ = oracle_mod.mstamp(T, meta["m"], meta["exclusion"])
    for (i, k, p, ok) in rows:
        assert abs(P[k, i] - p) < 1e-6, (i, k, P[k, i], p)
        assert int(I[k, i]) in ok, (i, k, I[k, i], ok)


# ---------------------------------------------------------------- invariants
@pytest.fixture(scope="module")
def c1(oracle_mod):
    cfg = datagen.make("C1")
    P, I, P2 = oracle_mod.mstamp(cfg["T"], cfg["m"], cfg["exclusion"])
    return cfg, P, I, P2


def test_bound(c1):
    """0 <= D'' <= 2 sqrt(m), since rho in [-1, 1] (Eq. (1))."""
    cfg, P, _, _ = c1
    assert np.all(P >= 0) and np.all(P <= 2 * math.sqrt(cfg["m"]) + 1e-12)


def test_monotone_in_k(c1):
    """P[k] <= P[k+1]: adding a value >= the current mean cannot lower the mean (Eq. (2))."""
    _, P, _, _ = c1
    assert np.all(np.diff(P, axis=0) >= -1e-12)


def test_symmetry_self_join(oracle_mod, c1):
    """Self-join: D''(i,j) = D''(j,i) bit-exactly, hence P[k][I[k][i]] <= P[k][i]."""
    cfg, P, I, _ = c1
    T, m = cfg["T"], cfg["m"]
    for (i, j) in [(5, 900), (1000, 33), (4095, 0)]:
        assert np.array_equal(oracle_mod.cell(T, m, i, j), oracle_mod.cell(T, m, j, i))
    d, n = P.shape
    for k in range(d):
        assert np.all(P[k, I[k]] <= P[k] + 1e-15)


def test_planted_motif(c1):
    """Embedded-motif recovery: I[k][a] = b, I[k][b] = a, P ~ 0 for k < k'."""
    cfg, P, I, _ = c1
    a, b = datagen.motif_positions(cfg["n"], cfg["m"])
    kk = max(1, cfg["d"] // 2)
    for k in range(kk):
        assert I[k, a] == b and I[k, b] == a
        assert P[k, a] < 1e-6 and P[k, b] < 1e-6


def test_dimension_permutation_bit_exact(oracle_mod):
    """The sort over dimensions (Eq. (2)) makes P, I invariant under permuting dimensions."""
    T = datagen.random_walk(5, 300, 16, 21)
    P, I, _ = oracle_mod.mstamp(T, 16, 4)
    Pp, Ip, _ = oracle_mod.mstamp(T[[3, 0, 4, 2, 1]], 16, 4)
    assert np.array_equal(P, Pp) and np.array_equal(I, Ip)


def test_power_of_two_scale_bit_exact(oracle_mod):
    """z-normalisation is scale invariant; a power-of-two scale is exact in FP (reading G16)."""
    T = datagen.random_walk(4, 300, 16, 22)
    P, I, _ = oracle_mod.mstamp(T, 16, 4)
    S = T * np.array([2.0 ** -7, 2.0 ** 3, 1.0, 2.0 ** -20])[:, None]
    Ps, Is, _ = oracle_mod.mstamp(S, 16, 4)
    assert np.array_equal(P, Ps) and np.array_equal(I, Is)


def test_affine_invariance(oracle_mod):
    T = datagen.random_walk(3, 250, 16, 23)
    P, I, _ = oracle_mod.mstamp(T, 16, 4)
    Pa, Ia, _ = oracle_mod.mstamp(3.7 * T - 123.25, 16, 4)
    assert np.array_equal(I, Ia) and np.allclose(P, Pa, rtol=1e-10, atol=1e-6)


def test_k0_is_min_of_1d_profiles(oracle_mod):
    """P[0][i] = min over dimensions of the classic 1-D matrix profile (textbook STOMP/MASS via FFT)."""
    T = datagen.random_walk(3, 400, 24, 24)
    P, _, _ = oracle_mod.mstamp(T, 24, 6)
    one_d = np.stack([brute.mass_1d(T[k], 24, 6) for k in range(3)])
    assert np.allclose(P[0], one_d.min(axis=0), rtol=1e-8, atol=1e-5)  # FFT rho error ~1e-14 -> D floor


def test_d1_is_1d_profile(oracle_mod):
    x = datagen.random_walk(1, 500, 32, 25)
    P, _, _ = oracle_mod.mstamp(x, 32, 8)
    assert np.allclose(P[0], brute.mass_1d(x[0], 32, 8), rtol=1e-8, atol=1e-5)


def test_last_k_is_plain_mean(oracle_mod):
    """P[d-1][i] = min_j of the plain mean over all dimensions (no sort needed)."""
    T = datagen.random_walk(4, 200, 16, 26)
    P, _, _ = oracle_mod.mstamp(T, 16, 4)
    D = brute.dist_cube(T, 16)
    M = D.mean(axis=0)
    n = M.shape[0]
    for i in range(n):
        M[i, max(0, i - 4):i + 5] = np.inf
    assert np.allclose(P[-1], M.min(axis=1), rtol=1e-12, atol=1e-12)


def test_exclusion_covers_everything(oracle_mod):
    """Reading G3: no admissible j -> P = +inf, I = -1."""
    T = datagen.random_walk(2, 20, 8, 27)
    P, I, P2 = oracle_mod.mstamp(T, 8, 19)
    assert np.all(np.isinf(P)) and np.all(I == -1)
    P, I, _ = oracle_mod.mstamp(T, 8, 17)   # only |i-j| = 18, 19 remain
    assert np.isinf(P[0, 5]) and I[0, 5] == -1 and np.isfinite(P[0, 0]) and I[0, 0] in (18, 19)


def test_flat_window_convention(oracle_mod):
    """Reading G4: a constant window has rho = 0 against everything -> D = sqrt(2m)."""
    m = 8
    T = datagen.random_walk(1, 100, m, 28)
    T[0, 40:40 + m] = 5.0
    out = oracle_mod.cell(T, m, 40, 80)
    assert out[0] == math.sqrt(2 * m)


def test_flat_windows_vs_bruteforce(oracle_mod):
    """Whole profiles with flat runs (several flat windows in a row, flat against flat, flat in one
    dimension only) against the brute force with G4 applied explicitly."""
    d, n, m, e = 2, 120, 8, 2
    T = datagen.random_walk(d, n, m, 42, motif=False)
    T[0, 20:40] = 1.5      # 13 consecutive flat windows in dim 0
    T[0, 80:90] = -2.0     # 3 more, far away (flat vs flat cells)
    T[1, 60:70] = 0.25
    P, I, P2 = oracle_mod.mstamp(T, m, e)
    Pb, Ib, P2b = brute.mstamp(T, m, e)
    assert np.all(np.abs(P - Pb) <= _near_tol(Pb, m, rtol=1e-11) + 1e-13)
    assert np.all(np.abs(P2 - P2b) <= _near_tol(P2b, m, rtol=1e-11) + 1e-13)
    _check_index(P, I, P2, Ib, Pb, 1e-9)
    assert np.allclose(brute.dist_cube(T, m)[0, 21, 81], math.sqrt(2 * m))


def test_sampled_rows_equal_full(oracle_mod, c1):
    cfg, P, I, P2 = c1
    rows = np.array([0, 17, 1041, 3043, 4095])
    Ps, Is, P2s = oracle_mod.mstamp(cfg["T"], cfg["m"], cfg["exclusion"], rows=rows)
    assert np.array_equal(Ps, P[:, rows]) and np.array_equal(Is, I[:, rows])
    assert np.array_equal(P2s, P2[:, rows])


def test_window_stats_two_pass(oracle_mod):
    T = datagen.random_walk(2, 100, 16, 29)
    mu, nrm = oracle_mod.window_stats(T, 16)
    w = np.lib.stride_tricks.sliding_window_view(T, 16, axis=1)
    assert np.allclose(mu, w.mean(axis=2), rtol=1e-15, atol=1e-12)
    assert np.allclose(nrm, np.sqrt(16) * w.std(axis=2), rtol=1e-13)


# ---------------------------------------------------------------- reading G7 (GPU-side recurrence)
def test_reading_g7_recurrence_identity():
    """The df/dg reading of Eq. (1) ("we do not repeat the equations")
    reproduces the direct centred dot products exactly in real arithmetic.  This pins the reading
    the CUDA path implements; it is test code, independent of both the oracle and the kernels."""
    m = 16
    x = datagen.random_walk(1, 300, m, 30)[0]
    y = datagen.random_walk(1, 300, m, 31)[0]
    wx = np.lib.stride_tricks.sliding_window_view(x, m)
    wy = np.lib.stride_tricks.sliding_window_view(y, m)
    mx, my = wx.mean(1), wy.mean(1)
    QT = (wx - mx[:, None]) @ (wy - my[:, None]).T

    def dfdg(v, mu):
        n = len(mu)
        df = np.zeros(n)
        dg = np.zeros(n)
        df[1:] = (v[m:m + n - 1] - v[:n - 1]) / 2.0
        dg[1:] = (v[m:m + n - 1] - mu[1:]) + (v[:n - 1] - mu[:-1])
        return df, dg

    dfx, dgx = dfdg(x, mx)
    dfy, dgy = dfdg(y, my)
    n = len(mx)
    for delta in (-100, -3, 0, 5, 170):
        i0, j0 = max(0, -delta), max(0, delta)
        q = QT[i0, j0]
        for s in range(1, n - max(i0, j0)):
            i, j = i0 + s, j0 + s
            q = q + dfx[i] * dgy[j] + dfy[j] * dgx[i]
            assert abs(q - QT[i, j]) <= 1e-9 * (1 + abs(QT[i, j]))


# ---------------------------------------------------------------- band partials
def _lexmin(parts):
    """(value, index) lexicographic min over band partials (the MINLOC merge, reading G2)."""
    P = np.full_like(parts[0][0], np.inf)
    I = np.full_like(parts[0][1], -1)
    for Pb, Ib in parts:
        Ib_key = np.where(Ib < 0, np.iinfo(np.int64).max, Ib)
        I_key = np.where(I < 0, np.iinfo(np.int64).max, I)
        take = (Pb < P) | ((Pb == P) & (Ib_key < I_key))
        P = np.where(take, Pb, P)
        I = np.where(take, Ib, I)
    return P, I


@pytest.mark.parametrize("ab", [False, True])
def test_band_all_diagonals_equals_rows(oracle_mod, ab):
    """A band covering every diagonal is the sampled-row profile, bit for bit."""
    d, n, m, e = 3, 300, 16, 4
    if ab:
        T, Tr = datagen.random_walk_ab(d, n, m, 61)
        dlo, dhi = -(n - 1), n
    else:
        T, Tr = datagen.random_walk(d, n, m, 61), None
        dlo, dhi = e + 1, n
    rows = np.arange(0, n, 7)
    P, I, P2 = oracle_mod.mstamp(T, m, e, Tr=Tr, rows=rows)
    Pb, Ib, P2b = oracle_mod.mstamp_band(T, m, rows, dlo, dhi, e, Tr=Tr)
    assert np.array_equal(P, Pb) and np.array_equal(I, Ib) and np.array_equal(P2, P2b)


@pytest.mark.parametrize("ab", [False, True])
def test_band_partition_merges_to_full(oracle_mod, ab):
    """Disjoint bands merged by lexicographic (value, index) min give the full profile."""
    d, n, m, e = 4, 260, 12, 3
    if ab:
        T, Tr = datagen.random_walk_ab(d, n, m, 62)
        cuts = [-(n - 1), -40, 0, 1, 90, n]
    else:
        T, Tr = datagen.random_walk(d, n, m, 62), None
        cuts = [e + 1, 9, 60, 61, n]
    rows = np.arange(n)
    P, I, _ = oracle_mod.mstamp(T, m, e, Tr=Tr)
    parts = [oracle_mod.mstamp_band(T, m, rows, a, b, e, Tr=Tr)[:2] for a, b in zip(cuts[:-1], cuts[1:])]
    Pm, Im = _lexmin(parts)
    assert np.array_equal(Pm, P) and np.array_equal(Im, I)


def test_band_vs_bruteforce(oracle_mod):
    """One band against the definitional brute force restricted to the band's cells."""
    d, n, m, e = 3, 90, 10, 2
    T = datagen.random_walk(d, n, m, 63, motif=False)
    D = brute.dist_cube(T, m)
    dlo, dhi = 20, 45
    rows = np.arange(n)
    Pb, Ib, _ = oracle_mod.mstamp_band(T, m, rows, dlo, dhi, e)
    for i in range(n):
        best = np.full(d, np.inf)
        for j in range(n):
            if not (dlo <= abs(j - i) < dhi) or abs(i - j) <= e:
                continue
            s = np.cumsum(np.sort(D[:, i, j])) / np.arange(1, d + 1)
            best = np.minimum(best, s)
        fin = np.isfinite(best)
        assert np.array_equal(fin, np.isfinite(Pb[:, i]))
        assert np.allclose(Pb[fin, i], best[fin], rtol=1e-11, atol=1e-12)
