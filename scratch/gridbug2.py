import os, sys, subprocess
sys.path.insert(0, "/root/repo")
import numpy as np, oracle
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
X = datagen.blobs(4096, 2, 6, noise=0.1, seed=1)
eps = 0.03
os.environ["EGGSYNC_SMALL"] = "0"
print("TC env", os.environ.get("EGGSYNC_TC"))
for t in range(1, 10):
    o = oracle.cluster(X, eps, max_iters=t)
    r = E.cluster(X, eps, coords=True, max_iters=t)
    d = np.abs(r["coords"] - o["X"]).max(axis=1)
    print(t, "maxdx %.2e" % d.max(), "bad points", int((d > 1e-5).sum()), np.nonzero(d > 1e-5)[0][:8], flush=True)
