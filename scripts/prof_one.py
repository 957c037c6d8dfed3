"""One hot-path call on a named config (for ncu captures): python scripts/prof_one.py C2 fp32 [reps]"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_juryl022_b200 import datagen, mstamp  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C2"
if name.startswith("X"):   # X<d>_<n>_<m>: ad-hoc self-join shape for profiling, e.g. X64_32768_256
    d_, n_, m_ = (int(v) for v in name[1:].split("_"))
    cfg = dict(T=datagen.random_walk(d_, n_, m_, 7), Tr=None, d=d_, n=n_, m=m_, exclusion=m_ // 4)
else:
    cfg = datagen.make(name)
prec = sys.argv[2] if len(sys.argv) > 2 else "fp32"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
d, n, m, e = cfg["d"], cfg["n"], cfg["m"], cfg["exclusion"]
T = torch.from_numpy(cfg["T"]).cuda()
Tr = None if cfg["Tr"] is None else torch.from_numpy(cfg["Tr"]).cuda()
P = torch.empty(d, n, dtype=torch.float64, device="cuda")
I = torch.empty(d, n, dtype=torch.int64, device="cuda")
ctx = mstamp.Context(0, seed_mode=os.environ.get("MP_SEED_MODE", "direct"))
import subprocess  # noqa: E402
for r in range(reps):
    ctx.compute_device(T, m, P, I, prec, e, Tr=Tr)
    ctx.compute_device(T, m, P, I, prec, e, Tr=Tr)
    clk = subprocess.run(["nvidia-smi", "--query-gpu=clocks.sm", "--format=csv,noheader,nounits"],
                         capture_output=True, text=True).stdout.strip()
    torch.cuda.synchronize()
    print(cfg["d"], n, prec, "main kernel ms", ctx.last_timing(), "sm_mhz(after)", clk)
