import os, sys
sys.path.insert(0, "/root/repo")
import numpy as np, oracle
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
X = datagen.blobs(4096, 2, 6, noise=0.1, seed=1)
eps = 0.03
o = oracle.cluster(X, eps)
print("oracle", o["rc"], o["iters"], o["labels"].max() + 1)
os.environ["EGGSYNC_SMALL"] = "0"
for tc in ["0", "2"]:
    pass
r = E.cluster(X, eps, coords=True)
print("grid", r["iters"], r["labels"].max() + 1, "labels equal", np.array_equal(r["labels"], o["labels"]),
      "maxdx", float(np.abs(r["coords"] - o["X"]).max()))
bad = np.nonzero(r["labels"] != o["labels"])[0]
print("mismatch idx", bad[:20], len(bad))
# step-by-step comparison
Xs = X.copy()
for t in range(r["iters"] + 1):
    g = E.step(Xs, eps, nbr=True)
    Xo, nb, f = oracle.step(Xs, eps, compute_f2=True)
    print(t, "nbr diff", int((g["nbr"] != nb).sum()), "maxdx %.2e" % float(np.abs(g["points"] - Xo).max()), "flags", g["first"], g["second"], f)
    Xs = g["points"]
