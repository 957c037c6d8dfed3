"""One diagonal band of a named config (mp_partial_device, rank of world), for ncu captures of
a representative share of a launch too long to replay whole:
python scripts/prof_band.py C3 fp32 7 16"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_ipps_juryl022_b200 import datagen, mstamp  # noqa: E402

name, prec = sys.argv[1], sys.argv[2]
rank, world = int(sys.argv[3]), int(sys.argv[4])
cfg = datagen.make(name)
d, n, m, e = cfg["d"], cfg["n"], cfg["m"], cfg["exclusion"]
T = torch.from_numpy(cfg["T"]).cuda()
Tr = None if cfg["Tr"] is None else torch.from_numpy(cfg["Tr"]).cuda()
keys = torch.empty(mstamp.key_words(d, n, prec), dtype=torch.int64, device="cuda")
ctx = mstamp.Context(0)
_, cells = mstamp.plan_bands(d, n, m, prec, e, cfg["Tr"] is None, world)
for r in range(2):
    ctx.partial_device(T, m, keys, rank, world, prec, e, Tr=Tr)
    torch.cuda.synchronize()
    print(name, prec, f"band {rank}/{world}", "cells", int(cells[rank]), "of", int(cells.sum()),
          "main kernel ms", ctx.last_timing())
