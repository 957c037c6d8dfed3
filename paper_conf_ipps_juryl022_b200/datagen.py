"""Seeded synthetic inputs shared by the oracle tests, the GPU parity tests and bench.py.

This module holds NO arithmetic of the method (no window statistics, no
distances, no sort/scan/min): it only draws numbers.  Both the oracle side and
the CUDA side consume its arrays; neither side's code lives here.

Recipe:
  * ``rng = np.random.default_rng(seed)``, steps ~ N(0, 1), ``T[k] = cumsum(steps[k])``,
    float64, shape (d, L), L = n + m - 1 -- random walks, the shape of the paper's
    stress-test series ("random noise combined with randomly-located
    injected repeating patterns").
  * One planted motif (the paper's embedded-pattern idea, PAPER.md:L911-915,
    L1218-1229): p[t] = 3 sin(2 pi 3 t / m) + 2 t / m, written continuity-preserving
    into dimensions 0..k'-1 (k' = max(1, d // 2)) at a = n//4 + 17 and b = 3n//4 - 29,
    i.e. T[k][x + t] - T[k][x - 1] = p[t].  Self-join: both copies in T.  AB-join:
    the copy at a in T_q, the copy at b in T_r (seed + 1000).
  * Bounded "paper-like" family: N(0,1) noise plus analogue shapes in [-1, 1]
    injected at random positions (used for FP16 error reporting).
"""
from __future__ import annotations

import numpy as np

CONFIGS = {
    # name: (join, d, n, m, exclusion, seed)   -- BASELINE.json configs C1..C5
    "C1": ("self", 4, 4096, 64, 16, 101),
    "C2": ("self", 16, 65536, 128, 32, 102),
    "C3": ("self", 64, 262144, 256, 64, 103),
    "C4": ("ab", 128, 1 << 20, 256, 0, 104),
    "C5": ("self", 256, 1 << 21, 512, 128, 105),
}


def motif_shape(m: int) -> np.ndarray:
    t = np.arange(m, dtype=np.float64)
    return 3.0 * np.sin(2.0 * np.pi * 3.0 * t / m) + 2.0 * (t / m)


def motif_positions(n: int, m: int):
    a = n // 4 + 17
    b = (3 * n) // 4 - 29
    if a < 1 or b < 1 or b + m > n + m - 1 or abs(a - b) <= m:
        return None
    return a, b


def _plant(steps: np.ndarray, x: int, p: np.ndarray, kk: int) -> None:
    # steps such that T[x+t] - T[x-1] == p[t]
    inc = np.empty_like(p)
    inc[0] = p[0]
    inc[1:] = np.diff(p)
    steps[:kk, x:x + len(p)] = inc


def random_walk(d: int, n: int, m: int, seed: int, motif: bool = True) -> np.ndarray:
    """(d, n+m-1) float64 random walk with an optional planted motif (self-join)."""
    L = n + m - 1
    rng = np.random.default_rng(seed)
    steps = rng.standard_normal((d, L))
    if motif:
        pos = motif_positions(n, m)
        if pos is not None:
            p = motif_shape(m)
            kk = max(1, d // 2)
            for x in pos:
                _plant(steps, x, p, kk)
    return np.cumsum(steps, axis=1)


def random_walk_ab(d: int, n: int, m: int, seed: int, motif: bool = True):
    """(T_q, T_r) for an AB-join; T_r uses seed + 1000; one shared motif."""
    L = n + m - 1
    rq = np.random.default_rng(seed).standard_normal((d, L))
    rr = np.random.default_rng(seed + 1000).standard_normal((d, L))
    if motif:
        pos = motif_positions(n, m)
        if pos is not None:
            p = motif_shape(m)
            kk = max(1, d // 2)
            _plant(rq, pos[0], p, kk)
            _plant(rr, pos[1], p, kk)
    return np.cumsum(rq, axis=1), np.cumsum(rr, axis=1)


PATTERN_NAMES = ["sine", "square", "triangle", "saw", "chirp", "gaussian", "step", "exp-decay"]


def pattern_shapes(m: int):
    """The eight analogue primitive shapes in [-1, 1] over t in [0, 1) (the paper's P0-P7 exist
    only as a drawing, Fig. 3; SURVEY 8(d) names these analogues)."""
    t = np.linspace(0.0, 1.0, m)
    return [np.sin(2 * np.pi * 2 * t), np.sign(np.sin(2 * np.pi * 2 * t)),
            2 * np.abs(2 * (2 * t % 1) - 1) - 1, 2 * (3 * t % 1) - 1,
            np.sin(2 * np.pi * (1 + 4 * t) * t), 2 * np.exp(-((t - 0.5) / 0.1) ** 2) - 1,
            np.where(t < 0.5, -1.0, 1.0), 2 * np.exp(-5 * t) - 1]


def embedded_pattern(d: int, n: int, m: int, shape: int, n_occ: int, seed: int, noise: float = 0.25):
    """(T, starts): N(0, noise^2) noise in d dims with pattern `shape` added at n_occ random,
    non-overlapping window starts (the paper's stress-test series with randomly located injected
    repeating patterns, and the embedded-motif recall set-up, L1218-1229)."""
    L = n + m - 1
    rng = np.random.default_rng(seed)
    T = noise * rng.standard_normal((d, L))
    p = pattern_shapes(m)[shape]
    starts = []
    while len(starts) < n_occ:
        x = int(rng.integers(0, n))
        if all(abs(x - y) >= 2 * m for y in starts):
            starts.append(x)
    for x in starts:
        T[:, x:x + m] += p
    return T, sorted(starts)


def bounded_patterns(d: int, n: int, m: int, seed: int, n_inject: int = 8) -> np.ndarray:
    """N(0,1) noise with analogue pattern shapes in [-1, 1] (paper-like bounded family)."""
    L = n + m - 1
    rng = np.random.default_rng(seed)
    T = 0.25 * rng.standard_normal((d, L))
    t = np.linspace(0.0, 1.0, m)
    shapes = [np.sin(2 * np.pi * 2 * t), np.sign(np.sin(2 * np.pi * 2 * t)),
              2 * np.abs(2 * (2 * t % 1) - 1) - 1, 2 * (3 * t % 1) - 1,
              np.sin(2 * np.pi * (1 + 4 * t) * t), 2 * np.exp(-((t - 0.5) / 0.1) ** 2) - 1,
              np.where(t < 0.5, -1.0, 1.0), 2 * np.exp(-5 * t) - 1]
    for k in range(d):
        for _ in range(n_inject):
            s = shapes[rng.integers(len(shapes))]
            x = int(rng.integers(0, L - m + 1))
            T[k, x:x + m] += s
    return T


def make(config: str):
    """Inputs of a named config: returns dict(T=..., Tr=None|..., d, n, m, exclusion)."""
    join, d, n, m, e, seed = CONFIGS[config]
    if join == "self":
        return dict(T=random_walk(d, n, m, seed), Tr=None, d=d, n=n, m=m, exclusion=e)
    Tq, Tr = random_walk_ab(d, n, m, seed)
    return dict(T=Tq, Tr=Tr, d=d, n=n, m=m, exclusion=0)
