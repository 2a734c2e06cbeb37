"""Two ranks driving the REAL library (not an oracle stand-in) through TorchComm.

Both processes share the one GPU of the test box (gloo backend, exchange staged through host
memory); each runs its own Context on its own stream, updates its block-interleaved owned
tiles with the kernel chosen from rank-reduced plan statistics, and all-gathers.  The result
must be bitwise identical to one process running the whole range (labels, iteration count,
coordinates): the multi-GPU scheme of DESIGN.md §8 ("replicate + own + all-gather").
"""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, X, eps, out):
    import torch
    import torch.distributed as dist
    from paper_conf_edbt_jorgensena23_b200 import distributed as DR
    from paper_conf_edbt_jorgensena23_b200 import eggsync as E
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        dev = torch.device("cuda", 0)
        s = torch.cuda.Stream(dev)
        torch.cuda.set_stream(s)
        n, d = X.shape
        ctx = E.Context(n, d, eps, device=0, stream=s.cuda_stream)
        ctx.load(X)
        comm = DR.TorchComm(n, d, dev, ctx=ctx)
        it, ok, lab = DR.run(ctx, comm)
        np.savez(os.path.join(out, f"r{rank}.npz"), it=it, ok=ok, lab=lab, X=ctx.coords())
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n,d,k,eps,noise", [(20000, 10, 6, 0.25, 0.05), (12000, 3, 5, 0.06, 0.0),
                                             (9000, 5, 4, 0.12, 0.1)])
def test_two_ranks_bitwise_equal_one(tmp_path, n, d, k, eps, noise):
    import torch.multiprocessing as mp
    from paper_conf_edbt_jorgensena23_b200 import datagen
    from paper_conf_edbt_jorgensena23_b200 import distributed as DR
    from paper_conf_edbt_jorgensena23_b200 import eggsync as E
    X = datagen.blobs(n, d, k, noise=noise, seed=3)
    ref = E.Context(n, d, eps)
    ref.load(X)
    it1, ok1, lab1 = DR.run(ref)
    X1 = ref.coords()
    mp.spawn(_worker, args=(2, _port(), X, eps, str(tmp_path)), nprocs=2, join=True)
    for r in range(2):
        g = np.load(tmp_path / f"r{r}.npz")
        assert bool(g["ok"]) == ok1 and int(g["it"]) == it1
        assert np.array_equal(g["lab"], lab1)
        assert np.array_equal(g["X"], X1), np.abs(g["X"] - X1).max()


def _worker_sharded(rank, world, port, X, eps, out):
    import torch
    import torch.distributed as dist
    from paper_conf_edbt_jorgensena23_b200 import distributed as DR
    from paper_conf_edbt_jorgensena23_b200 import eggsync as E
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        dev = torch.device("cuda", 0)
        s = torch.cuda.Stream(dev)
        torch.cuda.set_stream(s)
        n, d = X.shape
        share = np.array_split(np.arange(n), world)[rank]
        Xd = torch.from_numpy(X[share]).to(dev)
        ex = DR.ShardExchange(d, eps, dev)
        it, ok, lab, co = DR.run_sharded(Xd, torch.from_numpy(share.astype(np.int64)).to(dev), eps, ex,
                                         lambda m, dd: E.Context(m, dd, eps, device=0, stream=s.cuda_stream))
        if rank == 0:
            np.savez(os.path.join(out, "sh.npz"), it=it, ok=ok, lab=lab, X=co.cpu().numpy())
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("n,d,k,eps,noise", [(30000, 3, 6, 0.06, 0.02), (20000, 10, 5, 0.25, 0.05)])
def test_sharded_equals_one_gpu(tmp_path, world, n, d, k, eps, noise):
    """E2: no rank holds all points (slab shards + halo, own-point flags); labels and iteration
    count equal one GPU's, coordinates within the parity tolerance (local summation order)."""
    import torch.multiprocessing as mp
    from paper_conf_edbt_jorgensena23_b200 import datagen
    from paper_conf_edbt_jorgensena23_b200 import eggsync as E
    X = datagen.blobs(n, d, k, noise=noise, seed=5)
    ref = E.cluster(X, eps, coords=True)
    mp.spawn(_worker_sharded, args=(world, _port(), X, eps, str(tmp_path)), nprocs=world, join=True)
    g = np.load(tmp_path / "sh.npz")
    assert bool(g["ok"]) == ref["converged"] and int(g["it"]) == ref["iters"]
    assert np.array_equal(g["lab"], ref["labels"])
    assert np.abs(g["X"] - ref["coords"]).max() <= 1e-4
