# DEF42 (Def 4.2 literal, direct kernels) vs GRID clustering wall time, host input -> host labels
import os, sys, json, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
for cfg in sys.argv[1:] or ["C1", "C2"]:
    c = datagen.make_config(cfg)
    X = datagen.blobs(c.n, c.d, c.k, noise=c.noise, seed=0)
    out = {"cfg": cfg, "n": c.n, "d": c.d}
    for name, mode in (("grid", E.TERM_GRID), ("def42", E.TERM_DEF42)):
        E.cluster(X, c.eps, term_mode=mode)  # warm-up
        t = time.perf_counter(); r = E.cluster(X, c.eps, term_mode=mode); t = time.perf_counter() - t
        out[name] = {"s": t, "iters": r["iters"], "clusters": int(r["labels"].max()) + 1}
    print(json.dumps(out), flush=True)
