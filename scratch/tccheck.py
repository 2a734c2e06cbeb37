# dev check of the tensor-core update: small-case parity vs the oracle, C3 step TC vs SIMT, timings
import os, sys, time, json
sys.path.insert(0, "/root/repo")
import numpy as np
import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E

ok = True
for d in [int(x) for x in os.environ.get("DIMS", "2,3,5,10,16").split(",")]:
    for seed, (n, k, eps, noise) in enumerate([(3000, 4, 0.05, 0.0), (4000, 3, 0.08, 0.1)]):
        X = datagen.blobs(n, d, k, noise=noise, seed=seed)
        g = E.step(X, eps, nbr=True)
        Xo, nb, f = oracle.step(X, eps)
        dn = int((g["nbr"] != nb).sum())
        err = float(np.abs(g["points"] - Xo).max())
        s_ok = dn == 0 and err < 2e-6 and g["first"] == f[0]
        r = E.cluster(X, eps, coords=True)
        o = oracle.cluster(X, eps)
        c_ok = np.array_equal(r["labels"], o["labels"]) and r["iters"] == o["iters"] and np.abs(r["coords"] - o["X"]).max() < 1e-4
        print(f"d={d} n={n} step: nbr_mismatch={dn} maxerr={err:.2e} first={g['first']}/{f[0]} | cluster ok={c_ok} iters={r['iters']}/{o['iters']}", flush=True)
        ok &= s_ok and c_ok
print("SMALL_OK" if ok else "SMALL_FAIL", flush=True)

if os.environ.get("BIG", "1") == "1":
    c = datagen.make_config("C3")
    X = c.generate(0)
    for tc in ["1", "0"]:
        os.environ["EGGSYNC_TC"] = tc
    # step parity TC vs SIMT at full size (the env is read once per process: use the ctx flag)
    g = E.step(X, c.eps, nbr=True)
    print("C3 step TC first", g["first"], flush=True)
    E.cluster(X, c.eps)
    t = time.time()
    r = E.cluster(X, c.eps, stats=True)
    print("C3 cluster", r["iters"], "s", time.time() - t, json.dumps({k: v for k, v in r["stats"].items()}), flush=True)
    np.save("/root/repo/gpurun_out/c3_step_nbr_%s.npy" % os.environ.get("EGGSYNC_TC", "1"), g["nbr"])
    np.save("/root/repo/gpurun_out/c3_step_pts_%s.npy" % os.environ.get("EGGSYNC_TC", "1"), g["points"])
