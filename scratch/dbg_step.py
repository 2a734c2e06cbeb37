import numpy as np, sys
sys.path.insert(0, '/root/repo')
import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
for n in [3, 20, 40, 100, 1000]:
    X = datagen.blobs(n, 2, 2, seed=0)
    g = E.step(X, 0.05, nbr=True)
    Xo, nb, f = oracle.step(X, 0.05)
    ctx = E.Context(n, 2, 0.05); ctx.load(X); nc = ctx.build(); ctx.update(); ctx.advance(); Xc = ctx.coords()
    print(n, "ncells", nc, "nbr ok", np.array_equal(g["nbr"], nb), "max dx step", np.abs(g["points"] - Xo).max(), "ctx", np.abs(Xc - Xo).max())
    if n <= 40:
        print(" gpu", g["nbr"]); print(" ora", nb)
