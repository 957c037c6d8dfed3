"""Tier-0 definitional brute force (test helper; pins the C oracle).

Independent of the oracle's formula: it z-normalises every window explicitly
((x - mean) / population std) and takes the Euclidean distance between the
normalised windows -- the definition PAPER.md:L469 names ("Z-normalized
Euclidian distance") -- instead of sqrt(2m(1 - rho)) (Eq. (1)).  The two agree in
real arithmetic; agreement to ~1e-12 pins the oracle's Eq. (1) arithmetic.
Reading G4 (a flat window, norm 0, has rho = 0 against everything, so D = sqrt(2m)) is
applied explicitly: any cell with a flat window on either side gets D = sqrt(2m).  (Plain
z-normalisation to all-zeros would give sqrt(m) against a non-flat window and 0 between
two flat ones, which is not G4.)
"""
import numpy as np


def znorm_windows(x, m):
    """(z-normalised windows, flat mask); flat windows are left as zeros and masked."""
    w = np.lib.stride_tricks.sliding_window_view(x, m)
    mu = w.mean(axis=1, keepdims=True)
    sd = w.std(axis=1, keepdims=True)
    z = np.where(sd > 0, (w - mu) / np.where(sd > 0, sd, 1.0), 0.0)
    return z, sd[:, 0] == 0


def dist_cube(T, m, Tr=None):
    """D[k, i, j] z-normalised Euclidean distances (dense; tiny inputs only); G4 for flat windows."""
    Tr = T if Tr is None else Tr
    d = T.shape[0]
    out = []
    for k in range(d):
        zq, fq = znorm_windows(T[k], m)
        zr, fr = znorm_windows(Tr[k], m)
        diff = zq[:, None, :] - zr[None, :, :]
        D = np.sqrt((diff * diff).sum(axis=2))
        out.append(np.where(fq[:, None] | fr[None, :], np.sqrt(2.0 * m), D))
    return np.stack(out)


def mstamp(T, m, exclusion, Tr=None):
    """Returns P (d,n), I (d,n), P2 (d,n) by sorting each cell's d distances (Python sorted).

    P2[k][i] is the runner-up: the smallest D''_k(i, j) over admissible j other than I[k][i]
    (so P2 == P when another j ties the minimum exactly); +inf when fewer than two j exist."""
    D = dist_cube(T, m, Tr)
    d, n, _ = D.shape
    P = np.full((d, n), np.inf)
    P2 = np.full((d, n), np.inf)
    I = np.full((d, n), -1, dtype=np.int64)
    for i in range(n):
        vals = []
        for j in range(n):
            if Tr is None and abs(i - j) <= exclusion:
                continue
            s = sorted(D[:, i, j].tolist())
            acc = 0.0
            row = []
            for k in range(d):
                acc += s[k]
                row.append(acc / (k + 1))
            vals.append((j, row))
        for k in range(d):
            # lowest value, then lowest j (reading G2); the runner-up is the next entry
            ranked = sorted((row[k], j) for j, row in vals)
            if ranked:
                P[k, i], I[k, i] = ranked[0]
            if len(ranked) > 1:
                P2[k, i] = ranked[1][0]
    return P, I, P2


def mass_1d(x, m, exclusion, xr=None):
    """Classic 1-D matrix profile via FFT sliding dot products (MASS, textbook STOMP form).

    D^2 = 2m (1 - (QT - m mu_i mu_j) / (m sd_i sd_j)); a library FFT is the only step.
    """
    self = xr is None
    xr = x if self else xr
    L = len(x)
    n = L - m + 1
    wq = np.lib.stride_tricks.sliding_window_view(x, m)
    wr = np.lib.stride_tricks.sliding_window_view(xr, m)
    muq, sdq = wq.mean(1), wq.std(1)
    mur, sdr = wr.mean(1), wr.std(1)
    nfft = 1 << int(np.ceil(np.log2(2 * L)))
    FR = np.fft.rfft(xr, nfft)
    P = np.full(n, np.inf)
    for i in range(n):
        q = x[i:i + m][::-1]
        qt = np.fft.irfft(np.fft.rfft(q, nfft) * FR, nfft)[m - 1:m - 1 + n]
        rho = (qt - m * muq[i] * mur) / (m * sdq[i] * sdr)
        rho = np.clip(rho, -1, 1)
        dd = np.sqrt(2 * m * (1 - rho))
        if self:
            lo, hi = max(0, i - exclusion), min(n, i + exclusion + 1)
            dd[lo:hi] = np.inf
        P[i] = dd.min()
    return P
