"""Embedded-motif recall per pattern shape and precision mode (the paper's Fig. 3 analogue,
PAPER.md:L911-931, L1218-1262).

For each of the eight analogue shapes (datagen.pattern_shapes) a series of N(0, 0.25^2) noise in
d dimensions carries the shape at K random non-overlapping window starts (all dims).  For every
occurrence start x and every dimension count k, the matrix-profile index I[k][x] must point at
ANOTHER occurrence of the pattern:
  R_embedded      strict: I[k][x] is another occurrence's start,
  R^r_embedded    relaxed with factor r: within r*m of another occurrence's start (L917-931).
Modes: FP64 (the reference), FP32, Mixed, FP16CK, FP16C, FP16.  Writes profiles/r2_embedded_recall.json.
    python scripts/embedded_recall.py
"""
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_ipps_juryl022_b200 import datagen, mstamp  # noqa: E402

MODES = ["fp64", "fp32", "mixed", "fp16ck", "fp16c", "fp16"]
RELAX = [0.0, 0.01, 0.05, 0.1]


def recall(I, starts, m, r):
    """Fraction of (k, occurrence) pairs whose index lies within r*m of another occurrence."""
    st = np.asarray(starts)
    hits = tot = 0
    for x in starts:
        others = st[st != x]
        j = I[:, x]
        ok = (np.abs(j[:, None] - others[None, :]) <= r * m).any(axis=1)
        hits += int(ok.sum())
        tot += len(j)
    return hits / tot


def run(ctx, d, n, m, n_occ, seeds):
    out = {}
    for shape, name in enumerate(datagen.PATTERN_NAMES):
        acc = {mode: {r: [] for r in RELAX} for mode in MODES}
        for seed in seeds:
            T, starts = datagen.embedded_pattern(d, n, m, shape, n_occ, seed)
            for mode in MODES:
                _, I = ctx.compute(T, m, mode, m // 4)
                for r in RELAX:
                    acc[mode][r].append(recall(I, starts, m, r))
        out[name] = {mode: {f"r={r}": float(np.mean(v)) for r, v in acc[mode].items()} for mode in MODES}
    return out


def main():
    ctx = mstamp.Context(0)
    res = {"_doc": __doc__.split("\n\n")[0],
           "d16_n8192_m128_K8": run(ctx, 16, 8192, 128, 8, [1, 2, 3, 4]),
           "d64_n16384_m256_K8": run(ctx, 64, 16384, 256, 8, [5, 6])}
    ctx.close()
    with open(os.path.join(ROOT, "profiles", "r2_embedded_recall.json"), "w") as f:
        json.dump(res, f, indent=1)
    for cfg, tab in res.items():
        if cfg.startswith("_"):
            continue
        print(cfg)
        print(f"  {'shape':10s} " + " ".join(f"{m:>17s}" for m in MODES) + "   (strict / r=0.05)")
        for name, row in tab.items():
            print(f"  {name:10s} " + " ".join(f"{row[m]['r=0.0']:8.3f}/{row[m]['r=0.05']:8.3f}" for m in MODES))


if __name__ == "__main__":
    main()
