# per-iteration device time of the update (and build) for one config; EGGSYNC_TC selects the kernel
import os, sys, json
sys.path.insert(0, "/root/repo")
import torch
from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
cfg = sys.argv[1] if len(sys.argv) > 1 else "C3"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
c = datagen.make_config(cfg); X = c.generate(0); n, d = X.shape
dev = torch.device("cuda", 0); s = torch.cuda.Stream(dev); torch.cuda.set_stream(s)
Xd = torch.from_numpy(X).to(dev)
ctx = E.Context(n, d, c.eps, device=0, stream=s.cuda_stream)
for r in range(reps):
    ctx.load(Xd); t = 0; out = []
    while True:
        e = [torch.cuda.Event(enable_timing=True) for _ in range(3)]
        e[0].record(s); ctx.build(); e[1].record(s); ctx.update(); e[2].record(s)
        f1 = ctx.flags()[0]
        if f1 == 1:
            ctx.second_term()
            f2 = ctx.flags()[1]
        else:
            f2 = -1
        torch.cuda.synchronize()
        out.append((round(e[0].elapsed_time(e[1]), 3), round(e[1].elapsed_time(e[2]), 3)))
        ctx.advance(); t += 1
        if (f1 == 1 and f2 == 1) or t > 50:
            break
    print(json.dumps({"cfg": cfg, "tc": os.environ.get("EGGSYNC_TC", "1"), "rep": r, "iters": t, "build_update_ms": out}), flush=True)
