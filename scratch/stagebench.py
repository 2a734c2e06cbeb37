# per-stage device times of one clustering (eggsync_cluster_ex stats): Table-1 columns
import os, sys, json
sys.path.insert(0, "/root/repo")
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
for cfg in sys.argv[1:]:
    c = datagen.make_config(cfg); X = c.generate(0)
    E.cluster(X, c.eps)
    r = E.cluster(X, c.eps, stats=True)
    s = r["stats"]
    print(json.dumps({"cfg": cfg, "iters": r["iters"], **{k: (round(v * 1e3, 3) if isinstance(v, float) else v) for k, v in s.items()}}))
