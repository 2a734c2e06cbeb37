"""E2 sharded driver (distributed.run_sharded) on CPU with gloo, world sizes 2 and 3.

The per-rank local context is an oracle-backed stand-in for eggsync.Context (test
infrastructure): it holds the rank's own points followed by its halo, applies the oracle's
Eq.1 step (L68) to all of them, and reports the criterion flags over the own points only
(eggsync_ctx_set_own).  The sharded run must reproduce the single-process oracle clustering:
identical labels and iteration count, coordinates within 1e-6 (the summation order of the
local steps differs).  This checks the slab partition, the halo radius (cells that matter to
an own point complete locally), the all-to-all exchange and the flag reductions.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen
from paper_conf_edbt_jorgensena23_b200 import distributed as DR


class LocalOracleCtx:
    def __init__(self, n, d, eps):
        self.n, self.d, self.eps = n, d, eps
        c = oracle.constants(eps, d)
        self.inv_cw, self.w, self.e2, self.ed2 = c["inv_cw"], int(c["w"]), c["eps2"], c["ed2"]
        self.n_own = n

    def load(self, X):
        self.X = np.asarray(X, np.float32).astype(np.float64)

    def set_own(self, k):
        self.n_own = k

    def _cells(self, X):
        cc = np.minimum(np.floor(X * self.inv_cw), self.w - 1).astype(np.int64)
        _, first, inv = np.unique(cc, axis=0, return_index=True, return_inverse=True)
        return inv.reshape(-1), first

    def build(self):
        self.cell, _ = self._cells(self.X)

    def update(self):
        X, own = self.X, self.n_own
        self.Xn, nbr, _ = oracle.step(X, self.eps)
        cnt = np.bincount(self.cell)
        self.f1 = int(np.all(nbr[:own] == cnt[self.cell[:own]]))

    def flags(self):
        return self.f1, getattr(self, "f2", -1)

    def second_term(self):
        X, own = self.X, self.n_own
        d2 = ((X[None] - X[:, None]) ** 2).sum(-1)
        half = d2 <= self.e2 / 4.0
        ok = True
        for p in range(own):
            for q in np.nonzero((d2[p] > self.e2) & (d2[p] <= self.ed2))[0]:
                lo, hi = X[half[q]].min(0), X[half[q]].max(0)
                t = np.maximum(np.maximum(lo - X[p], 0.0), X[p] - hi)
                if (t * t).sum() <= self.e2:
                    ok = False
        self.f2 = int(ok)

    def advance(self):
        self.X = self.Xn.astype(np.float32).astype(np.float64)

    def coords(self):
        return self.X.astype(np.float32)

    def labels(self):
        inv, first = self._cells(self.X)
        rep = first[inv]                      # smallest index of the point's cell
        order = np.unique(rep)                # representatives in increasing index order
        return np.searchsorted(order, rep).astype(np.int32)


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, X, eps, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        n, d = X.shape
        share = np.array_split(np.arange(n), world)[rank]
        ex = DR.ShardExchange(d, eps, "cpu")
        it, ok, lab, co = DR.run_sharded(torch.from_numpy(X[share]), torch.from_numpy(share.astype(np.int64)), eps, ex,
                                         lambda m, dd: LocalOracleCtx(m, dd, eps))
        if rank == 0:
            np.savez(out, it=it, ok=ok, lab=lab, co=np.asarray(co))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
@pytest.mark.parametrize("n,d,k,eps,seed", [(240, 2, 3, 0.08, 0), (180, 3, 4, 0.12, 1)])
def test_sharded_equals_oracle(tmp_path, world, n, d, k, eps, seed):
    X = datagen.blobs(n, d, k, noise=0.1, seed=seed)
    out = str(tmp_path / "r0.npz")
    mp.spawn(_worker, args=(world, _port(), X, eps, out), nprocs=world, join=True)
    g = np.load(out)
    o = oracle.cluster(X, eps)
    assert bool(g["ok"]) and int(g["it"]) == o["iters"]
    assert np.array_equal(g["lab"], o["labels"])
    assert np.abs(g["co"].astype(np.float64) - o["X"]).max() <= 1e-6
