# dev check of the tensor-core update on a d=10 dev build (EGGSYNC_LIB=...lib_d10.so): parity vs the
# oracle on small cases, C4-d10 full clustering vs its golden, C3 sampled first step, per-iteration timings
import os, sys, time, json
sys.path.insert(0, "/root/repo")
import numpy as np
import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E

ok = True
D = int(os.environ.get("D", "10"))
for seed, (n, k, eps, noise) in enumerate([(8000, 4, 0.2, 0.0), (6000, 3, 0.25, 0.1), (3000, 5, 0.3, 0.0), (5000, 2, 0.15, 0.3)]):
    X = datagen.blobs(n, D, k, noise=noise, seed=seed)
    g = E.step(X, eps, nbr=True)
    Xo, nb, f = oracle.step(X, eps)
    dn = int((g["nbr"] != nb).sum())
    err = float(np.abs(g["points"] - Xo).max())
    s_ok = dn == 0 and err < 2e-6 and g["first"] == f[0]
    r = E.cluster(X, eps, coords=True)
    o = oracle.cluster(X, eps)
    c_ok = np.array_equal(r["labels"], o["labels"]) and r["iters"] == o["iters"] and np.abs(r["coords"] - o["X"]).max() < 1e-4
    print(f"d={D} n={n} eps={eps} step: nbr_mismatch={dn} maxerr={err:.2e} first={g['first']}/{f[0]} | cluster ok={c_ok} iters={r['iters']}/{o['iters']}", flush=True)
    ok &= s_ok and c_ok
print("SMALL_OK" if ok else "SMALL_FAIL", flush=True)
if os.environ.get("BIG", "1") == "1" and D == 10:
    gold = np.load("/root/repo/tests/golden/full/C4-d10_s0.npz")
    c = datagen.make_config("C4-d10")
    X = c.generate(0)
    t = time.time()
    r = E.cluster(X, c.eps, coords=True)
    lab_ok = np.array_equal(r["labels"], gold["labels"])
    err = float(np.abs(r["coords"][gold["sample_idx"]] - gold["sample_X"]).max())
    print(f"C4-d10 vs golden: labels_equal={lab_ok} iters={r['iters']}/{int(gold['iters'])} maxerr={err:.2e} ({time.time()-t:.2f}s)", flush=True)
    c = datagen.make_config("C3")
    X = c.generate(0)
    g = E.step(X, c.eps, nbr=True)
    idx = np.random.default_rng(0).choice(len(X), 192, replace=False)
    Xs, ns = oracle.step_sample(X, c.eps, idx)
    print(f"C3 step sampled: nbr_equal={np.array_equal(g['nbr'][idx], ns)} maxerr={np.abs(g['points'][idx] - Xs).max():.2e}", flush=True)
