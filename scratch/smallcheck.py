# F1 one-launch path: parity vs the oracle (C1 seeds, worked examples, bridge), e2e timing of C1
import os, sys, time, json
sys.path.insert(0, "/root/repo")
import numpy as np
import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
ok = True
c = datagen.CONFIGS["C1"]
for seed in range(4):
    X = c.generate(seed)
    g = E.cluster(X, c.eps, coords=True)
    o = oracle.cluster(X, c.eps)
    good = np.array_equal(g["labels"], o["labels"]) and g["iters"] == o["iters"] and np.abs(g["coords"] - o["X"]).max() < 1e-4
    print("C1 seed", seed, good, g["iters"], o["iters"], float(np.abs(g["coords"] - o["X"]).max()), flush=True)
    ok &= good
for n, d, k, eps in [(3000, 3, 4, 0.08), (2000, 8, 5, 0.3), (4096, 2, 6, 0.03), (1, 2, 1, 0.05), (777, 5, 3, 0.15)]:
    X = datagen.blobs(n, d, k, seed=1)
    g = E.cluster(X, eps, coords=True)
    o = oracle.cluster(X, eps)
    good = np.array_equal(g["labels"], o["labels"]) and g["iters"] == o["iters"] and np.abs(g["coords"] - o["X"]).max() < 1e-4
    print("blobs", n, d, good, g["iters"], o["iters"], flush=True)
    ok &= good
B = datagen.bridge()
g = E.cluster(B, 0.05, coords=True)
o = oracle.cluster(B, 0.05)
print("bridge", np.array_equal(g["labels"], o["labels"]), g["iters"], o["iters"], flush=True)
print("SMALL_OK" if ok else "SMALL_FAIL")
X = c.generate(0)
for _ in range(20):
    E.cluster(X, c.eps)
ts = []
for _ in range(200):
    t0 = time.perf_counter(); E.cluster(X, c.eps); ts.append(time.perf_counter() - t0)
print(json.dumps({"C1_e2e_ms_median": 1e3 * float(np.median(ts)), "C1_e2e_ms_min": 1e3 * min(ts)}))
os.environ["EGGSYNC_SMALL"] = "0"
