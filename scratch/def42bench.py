# GRID vs DEF42 (Def 4.2 literal: on the grid, and on the direct all-pairs kernels) clustering wall
# time, host input -> host labels; DIRECT skipped above 200k points (O(n^2))
import os, sys, json, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
for cfg in sys.argv[1:] or ["C1", "C2"]:
    c = datagen.make_config(cfg)
    X = datagen.blobs(c.n, c.d, c.k, noise=c.noise, seed=0)
    out = {"cfg": cfg, "n": c.n, "d": c.d}
    for name, mode in (("grid", E.TERM_GRID), ("def42", E.TERM_DEF42), ("def42_direct", E.TERM_DEF42_DIRECT)):
        if mode == E.TERM_DEF42_DIRECT and c.n > 200000:
            continue
        E.cluster(X, c.eps, term_mode=mode)  # warm-up
        t = time.perf_counter(); r = E.cluster(X, c.eps, term_mode=mode); t = time.perf_counter() - t
        out[name] = {"s": t, "iters": r["iters"], "clusters": int(r["labels"].max()) + 1}
    print(json.dumps(out), flush=True)
