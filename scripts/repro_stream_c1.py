"""Repeated streamed runs of C1 against the in-memory result (debugging aid for mp_compute_stream)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

from paper_conf_ipps_juryl022_b200 import datagen, mstamp  # noqa: E402

cfg = datagen.make("C1")
ctx = mstamp.Context(0, reseed_h=[256, 256, 64, 64])
T, m, e = cfg["T"], cfg["m"], cfg["exclusion"]
prec = sys.argv[1] if len(sys.argv) > 1 else "fp64"
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 4
P0, I0 = ctx.compute(T, m, prec, e)
os.environ["MP_STREAM_ROWS"] = "1"
os.environ["MP_STREAM_DIAGS"] = sys.argv[2] if len(sys.argv) > 2 else "500"
for r in range(reps):
    try:
        P1, I1 = ctx.compute_stream(T, m, prec, e, device_bytes=1 << 30)
        print(prec, r, "ok", np.array_equal(P0, P1), np.array_equal(I0, I1), ctx.last_stream_info(), flush=True)
    except Exception as ex:
        print(prec, r, "ERR", ex, flush=True)
        break
