"""Where FP32 departs most from the FP64 path on one config, in units of the parity tolerance.

python scripts/fp32_err_map.py X64_32768_256 [H ...]   (top entries by err/tol, per H)"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import parity  # noqa: E402
from paper_conf_ipps_juryl022_b200 import datagen, mstamp  # noqa: E402

name = sys.argv[1]
hs = [int(v) for v in sys.argv[2:]] or [0]
if name.startswith("X"):
    d_, n_, m_ = (int(v) for v in name[1:].split("_"))
    cfg = dict(T=datagen.random_walk(d_, n_, m_, 7), Tr=None, d=d_, n=n_, m=m_, exclusion=m_ // 4)
else:
    cfg = datagen.make(name)
d, n, m, e = cfg["d"], cfg["n"], cfg["m"], cfg["exclusion"]
T = torch.from_numpy(cfg["T"]).cuda()
P0 = torch.empty(d, n, dtype=torch.float64, device="cuda")
I0 = torch.empty(d, n, dtype=torch.int64, device="cuda")
mstamp.Context(0).compute_device(T, m, P0, I0, "fp64", e)
p0, i0 = P0.cpu().numpy(), I0.cpu().numpy()
fin = np.isfinite(p0)
tol = parity.tol_of(np.where(fin, p0, 0.0), m, "fp32", P0_row=np.where(fin[0], p0[0], np.inf))
kap = parity.kappa(cfg["T"], m)
for h in hs:
    ctx = mstamp.Context(0, reseed_h=[0, h, 0, 0])
    P = torch.empty_like(P0)
    I = torch.empty_like(I0)
    ctx.compute_device(T, m, P, I, "fp32", e)
    pg, ig = P.cpu().numpy(), I.cpu().numpy()
    r = np.abs(np.where(fin, pg - p0, 0.0)) / tol
    print(f"{name} H={h}: err/tol max {r.max():.3f}, entries > 1: {(r > 1).sum()} of {fin.sum()}, "
          f"rows > 1: {(r > 1).any(axis=0).sum()}; rel err quantiles 50/99/100 % "
          f"{np.quantile(np.abs(pg - p0)[fin] / p0[fin], [0.5, 0.99, 1.0])}", flush=True)
    top = np.argsort(r.ravel())[::-1][:8]
    for f in top:
        k, i = divmod(int(f), n)
        j = i0[k, i]
        print(f"  k={k} i={i} P64={p0[k, i]:.6f} P32={pg[k, i]:.6f} rel={abs(pg[k, i] - p0[k, i]) / p0[k, i]:.2e} "
              f"err/tol={r[k, i]:.2f} I64={j} I32={ig[k, i]} P64[0,i]={p0[0, i]:.4f} "
              f"kappa_i={kap[i]:.2f} kappa_j={kap[j]:.2f}", flush=True)
