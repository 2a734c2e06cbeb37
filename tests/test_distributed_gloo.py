"""Host logic of the multi-GPU driver (distributed.py) on CPU with gloo, world_size 2.

The per-rank phase object here is an oracle-backed stand-in for
eggsync.Context (test infrastructure only): it exposes the same phase methods
(build / update(lo,hi) / flags / second_term(lo,hi) / pack_into / unpack_from /
labels / advance) with the oracle's arithmetic, so the test checks exactly
the driver's sharding, exchange and flag-reduction logic: the 2-rank run must
reproduce the single-process oracle clustering bit for bit.
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


class OracleCtx:
    """Phase API over the fp64 oracle (identity 'sorted order')."""

    def __init__(self, X, eps):
        self.X = np.asarray(X, np.float64).copy()
        self.n, self.d = self.X.shape
        self.eps = eps
        c = oracle.constants(eps, self.d)
        self.inv_cw, self.w = c["inv_cw"], int(c["w"])
        self.e2, self.ed2 = c["eps2"], c["ed2"]

    def _cells(self, X):
        cc = np.minimum(np.floor(X * self.inv_cw), self.w - 1).astype(np.int64)
        _, inv = np.unique(cc, axis=0, return_inverse=True)
        return inv.reshape(-1)

    def build(self):
        X = self.X
        self.Xn, nbr, _ = oracle.step(X, self.eps)
        cell = self._cells(X)
        cnt = np.bincount(cell)
        self.f1p = nbr == cnt[cell]
        d2 = ((X[None] - X[:, None]) ** 2).sum(-1)
        half = d2 <= self.e2 / 4.0
        lo = np.stack([X[half[q]].min(0) for q in range(self.n)])
        hi = np.stack([X[half[q]].max(0) for q in range(self.n)])
        f2p = np.ones(self.n, bool)
        for p in range(self.n):
            for q in np.nonzero((d2[p] > self.e2) & (d2[p] <= self.ed2))[0]:
                t = np.maximum(np.maximum(lo[q] - X[p], 0.0), X[p] - hi[q])
                if (t * t).sum() <= self.e2:
                    f2p[p] = False
        self.f2p = f2p
        self.cell = cell
        self.nxt = np.full_like(X, np.nan)
        self.f = [1, 1]
        self.checked = False
        return int(cnt.size)

    def update(self, lo, hi):
        self.nxt[lo:hi] = self.Xn[lo:hi]
        self.f[0] &= int(self.f1p[lo:hi].all())

    def second_term(self, lo, hi):
        self.checked = True
        self.f[1] &= int(self.f2p[lo:hi].all())

    def flags(self):
        return self.f[0], (self.f[1] if self.checked else -1)

    # block-interleaved ownership (same index map as the library, block size B)
    B = 8

    def owned_count(self, R):
        nb = -(-self.n // self.B)
        return -(-nb // R) * self.B

    def _owned_pos(self, r, R, cnt):
        k = np.arange(cnt)
        return ((k // self.B) * R + r) * self.B + k % self.B

    def plan_owned(self, r, R):  # the library's plan statistics: [entries, points, tiles, overflow, max cell, tc]
        return np.array([7 * (r + 1), 7 * (r + 1), r + 1, 0, 3, 1], np.int64)

    def update_planned(self, r, R, g):
        # every rank sees the same rank-reduced statistics (SUM of 0..2, MAX of 3..5)
        tot = sum(range(1, R + 1))
        assert list(g) == [7 * tot, 7 * tot, tot, 0, 3, 1], g
        self.update_owned(r, R)

    def update_owned(self, r, R):
        pos = self._owned_pos(r, R, self.owned_count(R))
        pos = pos[pos < self.n]
        self.nxt[pos] = self.Xn[pos]
        self.f[0] &= int(self.f1p[pos].all())

    def pack_owned_into(self, r, R, t):
        cnt = self.owned_count(R)
        pos = self._owned_pos(r, R, cnt)
        t.zero_()
        ok = pos < self.n
        t[:, np.nonzero(ok)[0]] = torch.from_numpy(self.nxt[pos[ok]].T.astype(np.float32))

    def unpack_owned_from(self, t, R):
        cnt = self.owned_count(R)
        g = t.numpy().astype(np.float64)
        for r in range(R):
            pos = self._owned_pos(r, R, cnt)
            ok = pos < self.n
            self.nxt[pos[ok]] = g[r][:, ok].T

    def pack_into(self, lo, cnt, t):
        t.zero_()
        k = max(0, min(cnt, self.n - lo))
        t[:, :k] = torch.from_numpy(self.nxt[lo:lo + k].T.astype(np.float32))

    def unpack_from(self, t, ranks, cnt):
        g = t.numpy().astype(np.float64)
        for r in range(ranks):
            k = max(0, min(cnt, self.n - r * cnt))
            self.nxt[r * cnt:r * cnt + k] = g[r, :, :k].T

    def labels(self):
        first = {}
        return np.array([first.setdefault(c, len(first)) for c in self.cell], np.int32)

    def advance(self):
        self.X = self.nxt.copy()


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, X, eps, out, mode):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        ctx = OracleCtx(X.astype(np.float32), eps)
        comm = DR.TorchComm(ctx.n, ctx.d, "cpu", mode=mode, ctx=ctx)
        it, ok, lab = DR.run(ctx, comm)
        out[rank] = (it, ok, lab.tolist(), ctx.X.tolist(), comm.lo, comm.hi)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("mode", ["interleaved", "contiguous"])
@pytest.mark.parametrize("n,d,k,eps,seed", [(60, 2, 3, 0.08, 0), (75, 3, 4, 0.12, 1)])
def test_two_rank_run_equals_single_process(n, d, k, eps, seed, mode):
    X = datagen.blobs(n, d, k, seed=seed)
    # exchange in fp32 (the library's state type): the single-process reference does the same
    ref = OracleCtx(X, eps)
    it_ref, ok_ref, lab_ref = DR.run(_Fp32State(ref))
    mgr = mp.Manager()
    out = mgr.dict()
    port = _free_port()
    mp.spawn(_worker, args=(2, port, X, eps, out, mode), nprocs=2, join=True)
    assert set(out.keys()) == {0, 1}
    (it0, ok0, lab0, X0, lo0, hi0), (it1, ok1, lab1, X1, lo1, hi1) = out[0], out[1]
    assert (lo0, hi0, lo1, hi1) == (0, (n + 1) // 2, (n + 1) // 2, n)
    assert ok0 and ok1 and ok_ref
    assert it0 == it1 == it_ref
    assert lab0 == lab1 == lab_ref.tolist()
    assert np.array_equal(np.array(X0), np.array(X1))
    assert np.array_equal(np.array(X0), ref.X)
    # and the partition is the oracle's clustering
    o = oracle.cluster(X, eps)
    assert lab_ref.tolist() == o["labels"].tolist()


class _Fp32State:
    """Single-rank reference with the same fp32 rounding of the exchanged state."""

    def __init__(self, ctx):
        self.c = ctx
        self.n, self.d = ctx.n, ctx.d

    def __getattr__(self, k):
        return getattr(self.c, k)

    def advance(self):
        self.c.X = self.c.nxt.astype(np.float32).astype(np.float64)


def test_local_comm_covers_everything():
    c = DR.LocalComm(10)
    assert (c.lo, c.hi, c.world) == (0, 10, 1) and c.reduce_min(0) == 0
