# one small case per invocation for compute-sanitizer: python scratch/sanitize_case.py <case>
import os, sys
sys.path.insert(0, "/root/repo")
import numpy as np
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
case = sys.argv[1]
if case == "c1_small":
    c = datagen.CONFIGS["C1"]; r = E.cluster(c.generate(0), c.eps)
elif case == "c1_grid":
    os.environ["EGGSYNC_SMALL"] = "0"; c = datagen.CONFIGS["C1"]; r = E.cluster(c.generate(0), c.eps)
elif case == "tc":
    os.environ["EGGSYNC_TC"] = "2"; r = E.cluster(datagen.blobs(20000, 10, 5, noise=0.05, seed=1), 0.25)
elif case == "simt":
    os.environ["EGGSYNC_TC"] = "0"; r = E.cluster(datagen.blobs(20000, 10, 5, noise=0.05, seed=1), 0.25)
elif case == "def42":
    r = E.cluster(datagen.blobs(3000, 3, 4, seed=2), 0.08, term_mode=E.TERM_DEF42)
elif case == "def42_direct":
    r = E.cluster(datagen.blobs(3000, 3, 4, seed=2), 0.08, term_mode=E.TERM_DEF42_DIRECT)
print(case, "iters", r["iters"], "clusters", int(r["labels"].max()) + 1)
