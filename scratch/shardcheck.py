import os, sys, socket, traceback
sys.path.insert(0, "/root/repo")
import numpy as np

def port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0)); return s.getsockname()[1]

def worker(rank, world, p, X, eps):
    import torch, torch.distributed as dist
    from paper_conf_edbt_jorgensena23_b200 import distributed as DR, eggsync as E
    os.environ["MASTER_ADDR"] = "127.0.0.1"; os.environ["MASTER_PORT"] = str(p)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0); dev = torch.device("cuda", 0)
        s = torch.cuda.Stream(dev); torch.cuda.set_stream(s)
        n, d = X.shape
        share = np.array_split(np.arange(n), world)[rank]
        ex = DR.ShardExchange(d, eps, dev)
        it, ok, lab, co = DR.run_sharded(torch.from_numpy(X[share]).to(dev), torch.from_numpy(share.astype(np.int64)).to(dev),
                                         eps, ex, lambda m, dd: E.Context(m, dd, eps, device=0, stream=s.cuda_stream))
        print("rank", rank, "done", it, ok, flush=True)
        if rank == 0:
            ref = E.cluster(X, eps, coords=True)
            print("ref", ref["iters"], "labels equal", np.array_equal(lab, ref["labels"]), "maxdx", float(np.abs(co.cpu().numpy() - ref["coords"]).max()), flush=True)
    except Exception:
        traceback.print_exc()
        sys.stdout.flush()
        raise
    finally:
        dist.destroy_process_group()

if __name__ == "__main__":
    import torch.multiprocessing as mp
    from paper_conf_edbt_jorgensena23_b200 import datagen
    X = datagen.blobs(30000, 3, 6, noise=0.02, seed=5)
    mp.spawn(worker, args=(2, port(), X, 0.06), nprocs=2, join=True)
