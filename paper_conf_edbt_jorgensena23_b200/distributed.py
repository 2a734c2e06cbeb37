"""Algorithm 4 over the phase API, single- or multi-rank.

Multi-GPU scheme ("replicate + own + all-gather"): every rank
holds all n points and builds the identical structure (the build is
deterministic: Morton keys, stable sort, integer summaries), updates only the
points it owns (Eq.1 is a Jacobi update, L68, so owned sets are independent
given D^t), then the ranks exchange their updated points with one all-gather
(NCCL over NVLink via torch.distributed) and AND-reduce the two criterion
flags.  The update kernel (tensor-core or SIMT) is chosen from plan statistics
summed over all ranks (``eggsync_ctx_plan`` + all-reduce +
``eggsync_ctx_update_planned``), i.e. exactly as one GPU chooses it, and every
128-point tile is computed the same way on any rank: the result is bitwise
identical to one GPU.

Ownership is block-interleaved by default: the update's 128-point blocks (the
tensor-core point tile) of the sorted order are dealt round-robin to the
ranks, so dense cluster cores and sparse noise are spread evenly (a contiguous
split gives one rank the dense core).  torch.distributed is plumbing only; all
arithmetic is in the library.

Streams: the library runs on the context's stream, the collectives on torch's
current stream; ``TorchComm`` orders them with explicit stream waits.
"""
from __future__ import annotations

import math


class LocalComm:
    """World size 1: the whole range, no exchange."""

    def __init__(self, n: int):
        self.rank, self.world, self.lo, self.hi, self.cnt = 0, 1, 0, n, n

    def reduce_min(self, v: int) -> int:
        return v

    def update(self, ctx) -> None:
        ctx.update(self.lo, self.hi)

    def exchange(self, ctx) -> None:
        pass


class TorchComm:
    """One rank of a torch.distributed group.

    mode "interleaved": update blocks b with b % world == rank (load balance);
    mode "contiguous" : rank r owns sorted positions [r*cnt, min(n, (r+1)*cnt)).
    The second criterion term is split contiguously in both modes.
    """

    def __init__(self, n: int, d: int, device, group=None, mode: str = "interleaved", ctx=None):
        import torch
        import torch.distributed as dist
        self.torch, self.dist, self.group, self.mode = torch, dist, group, mode
        self.device = torch.device(device)
        self.backend = dist.get_backend(group)
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        span = math.ceil(n / self.world)
        self.lo = min(n, self.rank * span)                  # contiguous share (second term)
        self.hi = min(n, self.lo + span)
        if mode == "interleaved":
            if ctx is None:
                raise ValueError("interleaved ownership needs the context (block size)")
            self.cnt = ctx.owned_count(self.world)
        elif mode == "contiguous":
            self.cnt = span
        else:
            raise ValueError(mode)
        self.send = torch.empty((d, self.cnt), dtype=torch.float32, device=device)
        # concatenated layout (world*d, cnt) == stacked (world, d, cnt) in memory (gloo needs the former)
        self.recv = torch.empty((self.world * d, self.cnt), dtype=torch.float32, device=device)
        self.flag = torch.zeros(1, dtype=torch.int32, device=device)

    def reduce_min(self, v: int) -> int:
        flag = self.flag if self.backend == "nccl" or self.device.type != "cuda" else self.flag.cpu()
        flag.fill_(int(v))
        self.dist.all_reduce(flag, op=self.dist.ReduceOp.MIN, group=self.group)
        return int(flag.item())

    def reduce_plan(self, stats):
        """SUM of the entry / point / tile counts, MAX of the flags (eggsync.h)."""
        torch = self.torch
        dev = self.device if self.device.type == "cuda" and self.backend == "nccl" else torch.device("cpu")
        t = torch.tensor(stats, dtype=torch.int64, device=dev)
        s, m = t[:3].clone(), t[3:].clone()
        self.dist.all_reduce(s, op=self.dist.ReduceOp.SUM, group=self.group)
        self.dist.all_reduce(m, op=self.dist.ReduceOp.MAX, group=self.group)
        return torch.cat([s, m]).cpu().numpy()

    def update(self, ctx) -> None:
        if self.mode == "interleaved":
            # the update kernel is chosen from plan statistics of all ranks, as one GPU would
            g = self.reduce_plan(ctx.plan_owned(self.rank, self.world))
            ctx.update_planned(self.rank, self.world, g)
        else:
            ctx.update(self.lo, self.hi)

    def exchange(self, ctx) -> None:
        torch = self.torch
        cuda = self.device.type == "cuda"
        if cuda:
            xs = torch.cuda.ExternalStream(ctx.stream(), device=self.device)  # the library's stream
            cs = torch.cuda.current_stream(self.device)                        # the collective's stream
        if self.mode == "interleaved":
            ctx.pack_owned_into(self.rank, self.world, self.send)
        else:
            ctx.pack_into(self.lo, self.cnt, self.send)
        if cuda:
            cs.wait_stream(xs)   # the all-gather reads `send` after the pack kernel
        if cuda and self.backend != "nccl":
            # gloo between processes that share a GPU (tests): stage the exchange through host memory
            recv = torch.empty(self.recv.shape, dtype=self.recv.dtype)
            self.dist.all_gather_into_tensor(recv, self.send.cpu(), group=self.group)
            self.recv.copy_(recv)
        else:
            self.dist.all_gather_into_tensor(self.recv, self.send, group=self.group)
        if cuda:
            xs.wait_stream(cs)   # the unpack kernel reads `recv` after the all-gather
        view = self.recv.view(self.world, -1, self.cnt)
        if self.mode == "interleaved":
            ctx.unpack_owned_from(view, self.world)
        else:
            ctx.unpack_from(view, self.world, self.cnt)


def run(ctx, comm=None, max_iters: int = 10000, hooks=None):
    """Iterate until the criterion holds on the state the update read (readings R6/R7).

    ctx   : eggsync.Context (or any object with the same phase methods)
    comm  : LocalComm / TorchComm (None = LocalComm)
    hooks : optional object with before_update() / after_update() (timing)
    Returns (iters, converged, labels).
    """
    comm = comm or LocalComm(ctx.n)
    t, synced, labels = 0, False, None
    while True:
        ctx.build()
        if hooks:
            hooks.before_update()
        comm.update(ctx)                                  # Alg 3 on the owned points
        if hooks:
            hooks.after_update()
        f1 = comm.reduce_min(ctx.flags()[0])              # first term (Alg 3 l.14-15)
        f2 = -1
        if f1 == 1:                                       # Alg 4 l.9-10
            ctx.second_term(comm.lo, comm.hi)
            f2 = comm.reduce_min(ctx.flags()[1])
        synced = f1 == 1 and f2 == 1
        comm.exchange(ctx)                                # all ranks get D^{t+1}
        if synced:
            labels = ctx.labels()                         # cells of the verified state (L256)
        ctx.advance()
        t += 1
        if synced or t >= max_iters:
            break
    if not synced:
        labels = ctx.labels()
    return t, synced, labels


# --------------------------------------------------------------------------------------
# E2: sharded points.  No rank holds all n points: each rank owns the
# points of one slab of the first coordinate (quantile splitters, rebalanced every
# iteration) and receives a halo -- the other ranks' points within HALO * eps of its slab.
# With HALO >= 1.5 + delta/eps every grid cell that matters for an own point is complete
# locally: a cell within eps(+delta) of an own point has all its points within eps/2 more
# (cell diagonal eps/2, L252), so the own points' neighbourhoods (Eq.1), their cells
# (first term, L248/L252) and the cells of their shell points (MBR(N_eps/2(q)) of the
# second term, L108-110) are exact; only the own points' criterion flags count
# (eggsync_ctx_set_own).  Per iteration: one all-to-all moving points to their owners plus
# halo copies, a local build + update on own + halo, MIN all-reduces of the flags.  The
# labels are the cells of the verified state, gathered to rank 0 and numbered there by the
# library (L256, R14).  Local trees differ from one GPU's, so the sums are summed in another
# order: results agree with one GPU within the parity tolerance, not bitwise.
# --------------------------------------------------------------------------------------
HALO = 1.6


class ShardExchange:
    """Data distribution of the sharded driver (torch.distributed plumbing only)."""

    def __init__(self, d: int, eps: float, device, group=None, sample: int = 4096):
        import torch
        import torch.distributed as dist
        self.torch, self.dist, self.group = torch, dist, group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        self.device = torch.device(device)
        self.backend = dist.get_backend(group)
        self.d, self.h, self.sample = d, HALO * float(eps), sample

    def _coll_dev(self):
        return self.device if (self.backend == "nccl" and self.device.type == "cuda") else self.torch.device("cpu")

    def _all_gather_1d(self, t):
        torch = self.torch
        dev = self._coll_dev()
        n = torch.tensor([t.numel()], dtype=torch.int64, device=dev)
        ns = [torch.zeros_like(n) for _ in range(self.world)]
        self.dist.all_gather(ns, n, group=self.group)
        m = int(max(int(x) for x in ns))
        buf = torch.zeros(m, dtype=t.dtype, device=dev)
        buf[: t.numel()] = t.to(dev)
        outs = [torch.zeros_like(buf) for _ in range(self.world)]
        self.dist.all_gather(outs, buf, group=self.group)
        return torch.cat([o[: int(k)] for o, k in zip(outs, ns)])

    def splitters(self, x0):
        """World-1 quantiles of the first coordinate over a sample of every rank's points."""
        torch = self.torch
        k = min(self.sample, x0.numel())
        idx = torch.linspace(0, max(x0.numel() - 1, 0), k, device=x0.device).long() if k else \
            torch.zeros(0, dtype=torch.long, device=x0.device)
        allx = self._all_gather_1d(torch.sort(x0)[0][idx].float()).sort()[0]
        if allx.numel() == 0:
            return torch.zeros(self.world - 1, device=x0.device)
        q = torch.linspace(0, allx.numel() - 1, self.world + 1)[1:-1].round().long()
        return allx[q.to(allx.device)].to(x0.device)

    def exchange(self, X, gid, split):
        """Own points to their slab owners and halo copies to every rank within self.h of them.
        Returns (own X, own gid, halo X, halo gid) on this rank."""
        torch = self.torch
        R, dev = self.world, X.device
        x0 = X[:, 0]
        lo = torch.cat([torch.full((1,), -1e30, device=dev), split.to(dev)])
        hi = torch.cat([split.to(dev), torch.full((1,), 1e30, device=dev)])
        owner = torch.searchsorted(split.to(dev).contiguous(), x0.contiguous(), right=True)
        parts, counts = [], []
        for r in range(R):
            own = owner == r
            halo = (~own) & (x0 >= lo[r] - self.h) & (x0 < hi[r] + self.h)
            for m in (own, halo):
                parts.append((X[m], gid[m]))
                counts.append(int(m.sum()))
        cnt = torch.tensor(counts, dtype=torch.int64, device=self._coll_dev())
        rcnt = torch.empty_like(cnt)
        self.dist.all_to_all_single(rcnt, cnt, group=self.group)
        send_x = torch.cat([p[0] for p in parts]).reshape(-1)
        send_g = torch.cat([p[1] for p in parts])
        ssz = [counts[2 * r] + counts[2 * r + 1] for r in range(R)]
        rc = rcnt.cpu().tolist()
        rsz = [rc[2 * r] + rc[2 * r + 1] for r in range(R)]
        cd = self._coll_dev()
        recv_x = torch.empty(sum(rsz) * self.d, dtype=X.dtype, device=cd)
        recv_g = torch.empty(sum(rsz), dtype=gid.dtype, device=cd)
        self.dist.all_to_all_single(recv_x, send_x.to(cd), [s * self.d for s in rsz], [s * self.d for s in ssz],
                                    group=self.group)
        self.dist.all_to_all_single(recv_g, send_g.to(cd), rsz, ssz, group=self.group)
        recv_x = recv_x.to(dev).reshape(-1, self.d)
        recv_g = recv_g.to(dev)
        own_m = torch.zeros(sum(rsz), dtype=torch.bool, device=dev)
        off = 0
        for r in range(R):
            own_m[off: off + rc[2 * r]] = True
            off += rsz[r]
        return recv_x[own_m], recv_g[own_m], recv_x[~own_m], recv_g[~own_m]

    def min(self, v: int) -> int:
        t = self.torch.tensor([int(v)], dtype=self.torch.int32, device=self._coll_dev())
        self.dist.all_reduce(t, op=self.dist.ReduceOp.MIN, group=self.group)
        return int(t.item())

    def gather0(self, X, gid):
        """All points (X, gid) to rank 0, ordered by gid (None on the other ranks)."""
        torch = self.torch
        xs = self._all_gather_1d(X.reshape(-1).float())
        gs = self._all_gather_1d(gid.long())
        if self.rank != 0:
            return None
        order = torch.argsort(gs)
        return xs.reshape(-1, self.d)[order.to(xs.device)], gs[order]


def run_sharded(X_own, gid_own, eps: float, ex: ShardExchange, make_ctx, max_iters: int = 10000):
    """Algorithm 4 (L258-278) over sharded points.

    X_own   : (n_r, d) float32 tensor, this rank's initial share of the points
    gid_own : (n_r,) int64 tensor, their global indices (0..n-1)
    make_ctx: callable(n_local, d) -> a context (eggsync.Context or a stand-in) for own + halo
    Returns (iters, converged, labels, coords) on rank 0 (labels / coords in global index
    order), (iters, converged, None, None) elsewhere.
    """
    torch = ex.torch
    d = ex.d
    X, gid = X_own, gid_own
    t, synced = 0, False
    verified = None
    while True:
        split = ex.splitters(X[:, 0])
        Xo, go, Xh, gh = ex.exchange(X, gid, split)
        n_own = Xo.shape[0]
        ctx = make_ctx(n_own + Xh.shape[0], d)
        loc = torch.cat([Xo, Xh]).contiguous()
        ctx.load(loc.cpu().numpy() if not loc.is_cuda else loc)
        ctx.set_own(n_own)
        ctx.build()
        ctx.update()
        f1 = ex.min(ctx.flags()[0])                        # first term over all own points
        f2 = -1
        if f1 == 1:
            ctx.second_term()
            f2 = ex.min(ctx.flags()[1])
        synced = f1 == 1 and f2 == 1
        ctx.advance()
        nxt = ctx.coords()
        nxt = torch.as_tensor(nxt, device=X.device)[:n_own]
        if synced:
            verified = (Xo, go)                            # D^t: its cells are the clusters (R7)
        X, gid = nxt, go
        t += 1
        if hasattr(ctx, "close"):
            ctx.close()
        if synced or t >= max_iters:
            break
    final = ex.gather0(X, gid)
    state = ex.gather0(*(verified if synced else (X, gid)))
    if ex.rank != 0:
        return t, synced, None, None
    Xs = state[0].contiguous()
    ctx = make_ctx(Xs.shape[0], d)
    ctx.load(Xs.cpu().numpy() if not Xs.is_cuda else Xs)
    ctx.build()
    labels = ctx.labels()                                  # cells of the verified state (L256)
    if hasattr(ctx, "close"):
        ctx.close()
    return t, synced, labels, final[0]
