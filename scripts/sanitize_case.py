"""One small hot-path call per kernel family, for compute-sanitizer (memcheck / racecheck /
synccheck): python scripts/sanitize_case.py <prec> <d> <self|ab> [n] [m]
No torch: the host-memory C-ABI entry point only."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_ipps_juryl022_b200 import datagen, mstamp  # noqa: E402

prec, d, join = sys.argv[1], int(sys.argv[2]), sys.argv[3]
n = int(sys.argv[4]) if len(sys.argv) > 4 else 300
m = int(sys.argv[5]) if len(sys.argv) > 5 else 16
ctx = mstamp.Context(0)
if join == "self":
    P, I = ctx.compute(datagen.random_walk(d, n, m, 5), m, prec, m // 4)
else:
    Tq, Tr = datagen.random_walk_ab(d, n, m, 6)
    P, I = ctx.compute(Tq, m, prec, Tr=Tr)
print(prec, d, join, "ok", float(P[0].min()))
ctx.close()
