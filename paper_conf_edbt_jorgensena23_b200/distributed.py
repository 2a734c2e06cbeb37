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
