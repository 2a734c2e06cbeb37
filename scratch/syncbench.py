# Direct (GPU-SynC-style) Eq.1 update vs the grid path, one update on device-resident input.
import os, sys, json, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
for cfg in sys.argv[1:] or ["C2", "C3"]:
    c = datagen.make_config(cfg)
    X = datagen.blobs(c.n, c.d, c.k, noise=c.noise, seed=0)
    t = torch.from_numpy(X).cuda()
    ts = []
    for r in range(3):
        u = t.clone(); torch.cuda.synchronize()
        a = time.perf_counter(); g = E.sync_step(u, c.eps); torch.cuda.synchronize()
        ts.append(time.perf_counter() - a)
    pairs = float(c.n) * c.n
    print(json.dumps({"cfg": cfg, "n": c.n, "d": c.d, "sync_step_s": ts, "rc": g["rc"],
                      "pairs_per_s": pairs / min(ts),
                      "alu_instr_per_s": pairs * (2 * c.d + 2) / min(ts)}), flush=True)
