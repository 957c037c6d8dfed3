"""Element-wise error of the half-precision modes (FP16, Mixed, FP16C; Fig. 1,
L773-798) over FULL grids: the distribution of |P - P64| / sqrt(2m) over every (k, i), P64 the
GPU FP64 path (within 1e-9 of the oracle, tests/test_gpu_parity.py), and the same quantity
against the FP64 oracle itself on sampled rows.  sqrt(2m) is the distance of two uncorrelated
z-normalised windows (rho = 0), so the figure is the error in units of the distance scale.
Writes profiles/r2_half_bounds.json (the bounds stated in DESIGN.md section 7 and asserted by
tests/test_gpu_parity.py::test_half_modes_elementwise_bound).
    python scripts/half_bounds.py [C1 C2 C3]
"""
import json
import math
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import torch  # noqa: E402

import oracle  # noqa: E402  (test infrastructure: the checker, never the product path)
from paper_conf_ipps_juryl022_b200 import datagen, mstamp  # noqa: E402

MODES = ["mixed", "fp16ck", "fp16c", "fp16"]


def stats(err, scale):
    e = err / scale
    return {"max": float(e.max()), "p999": float(np.quantile(e, 0.999)), "p99": float(np.quantile(e, 0.99)),
            "median": float(np.median(e))}


def main():
    names = sys.argv[1:] or ["C1", "C2", "C3"]
    out = {}
    path = os.path.join(ROOT, "profiles", "r2_half_bounds.json")
    if os.path.exists(path):
        out = json.load(open(path))
    ctx = mstamp.Context(0)
    oracle.build()
    for name in names:
        cfg = datagen.make(name)
        T, m, e, n, d = cfg["T"], cfg["m"], cfg["exclusion"], cfg["n"], cfg["d"]
        Td = torch.from_numpy(T).cuda()
        P64 = torch.empty(d, n, dtype=torch.float64, device="cuda")
        I64 = torch.empty(d, n, dtype=torch.int64, device="cuda")
        ctx.compute_device(Td, m, P64, I64, "fp64", e)
        p64 = P64.cpu().numpy()
        i64 = I64.cpu().numpy()
        fin = np.isfinite(p64)
        rng = np.random.default_rng(11)
        a, b = datagen.motif_positions(n, m)
        rows = np.unique(np.concatenate([[0, n - 1, a, b], rng.integers(0, n, 24 if n > 8192 else 200)]))
        Po, Io, _ = oracle.mstamp(T, m, e, rows=rows)
        scale = math.sqrt(2 * m)
        for mode in MODES:
            P = torch.empty_like(P64)
            I = torch.empty_like(I64)
            ctx.compute_device(Td, m, P, I, mode, e)
            p, i = P.cpu().numpy(), I.cpu().numpy()
            rec = {"full_grid_vs_fp64": stats(np.abs(p - p64)[fin], scale),
                   "sampled_rows_vs_oracle": stats(np.abs(p[:, rows] - Po)[np.isfinite(Po)], scale),
                   "rows_sampled": int(len(rows)), "index_recall_vs_fp64": float(np.mean(i[fin] == i64[fin])),
                   "entries": int(fin.sum())}
            out[f"{name}/{mode}"] = rec
            print(name, mode, json.dumps(rec), flush=True)
        del Td, P64, I64
        torch.cuda.empty_cache()
    with open(path, "w") as f:
        json.dump(out, f, indent=1)


if __name__ == "__main__":
    main()
