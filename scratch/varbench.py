import os, sys, time, json
sys.path.insert(0, "/root/repo")
import numpy as np, torch
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E, distributed as DR
cfg = os.environ.get("CFG", "C3")
c = datagen.make_config(cfg); X = c.generate(0); n, d = X.shape
s = torch.cuda.Stream(); torch.cuda.set_stream(s)
Xd = torch.from_numpy(X).cuda()
ctx = E.Context(n, d, c.eps, device=0, stream=s.cuda_stream)
class H:
    def __init__(s_): s_.ev = []
    def before_update(s_):
        e = torch.cuda.Event(enable_timing=True); e.record(s); s_.ev.append([e, None])
    def after_update(s_):
        e = torch.cuda.Event(enable_timing=True); e.record(s); s_.ev[-1][1] = e
res = []
for rep in range(5):
    h = H(); ctx.load(Xd); torch.cuda.synchronize(); t0 = time.perf_counter()
    it, ok, lab = DR.run(ctx, hooks=h); torch.cuda.synchronize(); dt = time.perf_counter() - t0
    res.append((dt * 1e3, [a.elapsed_time(b) for a, b in h.ev]))
best = min(res, key=lambda r: r[0])
print(json.dumps({"lib": os.path.basename(os.environ.get("EGGSYNC_LIB", "default")), "cfg": cfg, "iters": it,
                  "step_ms": round(best[0], 2), "upd_ms": [round(x, 2) for x in best[1]]}))
