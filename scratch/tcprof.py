import sys, os
sys.path.insert(0, "/root/repo")
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
c = datagen.make_config(sys.argv[1] if len(sys.argv) > 1 else "C3")
X = c.generate(0)
r = E.cluster(X, c.eps)
print("iters", r["iters"])
