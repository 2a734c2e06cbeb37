# per-configuration clustering time with the radix tree (default) and the random-access grid
# (EGGSYNC_DENSE=1, d <= 4), device-resident input, one warm-up; each mode in its own process
import os, sys, json, time, subprocess
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
if len(sys.argv) > 1 and sys.argv[1] == "--one":
    import torch
    from paper_conf_edbt_jorgensena23_b200 import datagen, eggsync as E
    out = {}
    for cfg in sys.argv[2:]:
        c = datagen.make_config(cfg)
        X = torch.from_numpy(c.generate(0)).cuda()
        E.cluster(X, c.eps)
        torch.cuda.synchronize()
        t = time.perf_counter(); r = E.cluster(X, c.eps); torch.cuda.synchronize(); t = time.perf_counter() - t
        out[cfg] = {"s": t, "iters": r["iters"], "clusters": int(r["labels"].max().item()) + 1}
    print(json.dumps(out))
else:
    cfgs = sys.argv[1:] or ["C1", "C4-d2", "C5"]
    for mode in ("0", "1"):
        env = dict(os.environ, EGGSYNC_DENSE=mode)
        r = subprocess.run([sys.executable, __file__, "--one", *cfgs], env=env, capture_output=True, text=True)
        print(json.dumps({"dense": mode, "results": json.loads(r.stdout.strip().splitlines()[-1]) if r.returncode == 0 else r.stderr[-800:]}), flush=True)
