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
