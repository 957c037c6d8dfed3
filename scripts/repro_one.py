import sys; sys.path.insert(0,'/root/repo')
import numpy as np
from paper_conf_ipps_juryl022_b200 import datagen, mstamp
d,n,m,e,seed = [int(x) for x in sys.argv[1:6]]
prec = sys.argv[6]
T = datagen.random_walk(d, n, m, seed)
ctx = mstamp.Context(0)
P,I = ctx.compute(T, m, prec, e)
print("ok", d, n, m, prec, P[0,:3])
