import os, sys
sys.path.insert(0, "/root/repo")
import numpy as np
import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
d = int(sys.argv[1])
ok = True
for seed, (n, k, eps, noise) in enumerate([(3000, 4, 0.05, 0.0), (4000, 3, 0.08, 0.1), (2000, 6, 0.03, 0.0)]):
    X = datagen.blobs(n, d, k, noise=noise, seed=seed)
    g = E.step(X, eps, nbr=True); Xo, nb, f = oracle.step(X, eps)
    s_ok = np.array_equal(g["nbr"], nb) and np.abs(g["points"] - Xo).max() < 2e-6 and g["first"] == f[0]
    r = E.cluster(X, eps, coords=True); o = oracle.cluster(X, eps)
    c_ok = np.array_equal(r["labels"], o["labels"]) and r["iters"] == o["iters"] and np.abs(r["coords"] - o["X"]).max() < 1e-4
    print(f"d={d} n={n} sub={os.environ.get('EGGSYNC_SUBBITS','default')} step_ok={s_ok} cluster_ok={c_ok} iters={r['iters']}/{o['iters']}")
    ok &= s_ok and c_ok
print("ALL_OK" if ok else "FAIL")
