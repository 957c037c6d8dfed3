"""Re-seed interval sweep on one config: main-kernel time and error against FP64 per H.

python scripts/h_sweep.py C2 fp32 512,1024,2048
Error = max |P - P_fp64| / P_fp64 over finite entries (P_fp64 at the default FP64 interval)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

from paper_conf_ipps_juryl022_b200 import datagen, mstamp  # noqa: E402
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import parity  # noqa: E402

name, prec = sys.argv[1], sys.argv[2]
hs = [int(v) for v in sys.argv[3].split(",")]
if name.startswith("X"):   # X<d>_<n>_<m>: ad-hoc self-join shape
    d_, n_, m_ = (int(v) for v in name[1:].split("_"))
    cfg = dict(T=datagen.random_walk(d_, n_, m_, 7), Tr=None, d=d_, n=n_, m=m_, exclusion=m_ // 4)
else:
    cfg = datagen.make(name)
d, n, m, e = cfg["d"], cfg["n"], cfg["m"], cfg["exclusion"]
T = torch.from_numpy(cfg["T"]).cuda()
Tr = None if cfg["Tr"] is None else torch.from_numpy(cfg["Tr"]).cuda()
P0 = torch.empty(d, n, dtype=torch.float64, device="cuda")
I0 = torch.empty(d, n, dtype=torch.int64, device="cuda")
mstamp.Context(0).compute_device(T, m, P0, I0, "fp64", e, Tr=Tr)
slot = {"fp64": 0, "fp32": 1, "fp16": 2, "mixed": 3}[prec]
for h in hs:
    rh = [0, 0, 0, 0]
    rh[slot] = h
    ctx = mstamp.Context(0, reseed_h=rh)
    P = torch.empty_like(P0)
    I = torch.empty_like(I0)
    ts = []
    for _ in range(3):
        ctx.compute_device(T, m, P, I, prec, e, Tr=Tr)
        torch.cuda.synchronize()
        ts.append(ctx.last_timing()[0])
    ok = torch.isfinite(P0) & (P0 > 1e-6)
    err = ((P - P0).abs()[ok] / P0[ok]).max().item()
    # error in units of the parity tolerance (tests/parity.py; FP64 GPU result as reference)
    p0 = P0.cpu().numpy()
    fin = np.isfinite(p0)
    tol = parity.tol_of(np.where(fin, p0, 0.0), m, "fp64" if prec == "fp64" else "fp32",
                        P0_row=np.where(fin[0], p0[0], np.inf))
    ratio = float((np.abs(np.where(fin, P.cpu().numpy() - p0, 0.0)) / tol).max())
    same_i = (I == I0).float().mean().item()
    print(f"{name} {prec} H={h} main_ms={min(ts):.2f} max_rel_err={err:.3e} idx_agree={same_i:.4f} err/tol={ratio:.3f}", flush=True)
