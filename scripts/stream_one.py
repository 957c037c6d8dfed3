"""One beyond-memory streamed run (mp_compute_stream) of a named config with a device budget:
python scripts/stream_one.py C3 fp32 536870912  (MP_STREAM_PROFILE=1 prints host phase times)."""
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_ipps_juryl022_b200 import datagen, mstamp  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "C3"
prec = sys.argv[2] if len(sys.argv) > 2 else "fp32"
budget = int(sys.argv[3]) if len(sys.argv) > 3 else 512 << 20
if name.startswith("X"):   # X<d>_<n>_<m>: ad-hoc self-join shape
    d_, n_, m_ = (int(v) for v in name[1:].split("_"))
    cfg = dict(T=datagen.random_walk(d_, n_, m_, 7), Tr=None, m=m_, exclusion=m_ // 4)
else:
    cfg = datagen.make(name)
ctx = mstamp.Context(0)
T, Tr, m, e = cfg["T"], cfg["Tr"], cfg["m"], cfg["exclusion"]
for rep in range(int(os.environ.get("REPS", "2"))):
    t0 = time.perf_counter()
    P, I = ctx.compute_stream(T, m, prec, e, Tr=Tr, device_bytes=budget)
    dt = time.perf_counter() - t0
    R, Wb, peak, nl = ctx.last_stream_info()
    kms, _ = ctx.last_timing()
    print(f"{name} {prec} budget {budget >> 20} MiB: wall {dt * 1e3:.0f} ms, kernels {kms:.0f} ms, R {R} Wb {Wb} "
          f"peak {peak >> 20} MiB, launches {nl}", flush=True)
t0 = time.perf_counter()
P0, I0 = ctx.compute(T, m, prec, e, Tr=Tr)
print(f"in-memory mp_compute wall {(time.perf_counter() - t0) * 1e3:.0f} ms; bit-identical:",
      bool(np.array_equal(P, P0) and np.array_equal(I, I0)))
