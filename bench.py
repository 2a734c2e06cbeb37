#!/usr/bin/env python
"""Benchmark of the EGG-SynC synchronization update on B200 (BASELINE.json metric).

One step = one complete EGG-SynC clustering (all §8(a) rows: keys, sort, cell
offsets, summaries, hierarchy, update, both criterion terms, labels) of the
workload BASELINE.json's metric is quoted on: C3, n=1,000,000, d=10, 20
Gaussian clusters + 5% uniform noise, eps=0.1 (synthetic, seed 0).

  value  = point-updates/s = n * iters / device time of the step (inputs
           resident in HBM; L2 flushed by a 256 MiB write between steps)
  e2e    = the same metric through eggsync_cluster() with pinned HOST
           buffers (H2D of the points and D2H of the labels inside the timing)

Usage:  python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
        (N>1: launched under torch.distributed.run, one rank per GPU, NCCL)
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

METRIC = "end-to-end clustering sec and point-updates/sec at n=1M,d=10; 1/2/4/8 B200"
UNIT = "point-updates/s"
PEAKS_PATH = os.path.join(ROOT, "MEASURED_PEAKS.json")
SM_COUNT, FP32_LANES = 148, 128


def workload_desc(c):
    return (f"{c.name}: n={c.n:,} d={c.d} {c.k} Gaussian clusters (std 5 in [-100,100]^d)"
            f" + {int(c.noise * 100)}% uniform noise, min/max-normalised, eps={c.eps}, seed 0")


# ----------------------------------------------------------------- clocks
class ClockSampler:
    """nvidia-smi clocks and throttle reasons during the timed region (B200_PROFILING.md)."""

    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index, self.rows, self.proc = index, [], None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-i", str(self.index), "-lms", "200"], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 7:
                self.rows.append(parts)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": [], "samples": 0}
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in self.rows for k in range(4) if r[3 + k].lower() == "active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


# -------------------------------------------------------- cpu baseline
def oracle_rate(X, eps, target_s: float, seed: int = 0):
    """The fp64 oracle (as it stands) on a bounded sample: Eq.1 updates of m sampled points
    against the full state (oracle_step_sample).  Returns (point-updates/s, m, seconds, cores)."""
    import oracle
    rng = np.random.default_rng(seed)
    m = 8
    while True:
        idx = rng.choice(len(X), m, replace=False)
        t0 = time.perf_counter()
        oracle.step_sample(X, eps, idx)
        dt = time.perf_counter() - t0
        if dt >= 0.25 * target_s or m >= len(X):
            return m / dt, m, dt, os.cpu_count()
        m = int(min(len(X), max(m * 2, m * 0.3 * target_s / max(dt, 1e-3))))


def cpu_model() -> str:
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    import platform
    return platform.processor() or "unknown"


def cpu_baseline_obj(X, c, target_s):
    rate, m, dt, cores = oracle_rate(X, c.eps, target_s)
    return {"value": rate, "unit": UNIT, "cores": cores, "cpu_model": cpu_model(), "kind": "oracle",
            "sample": f"{m} Eq.1 point-updates of {c.name} iteration 1 (each against the full n={c.n:,} state), "
                      f"fp64 C/OpenMP oracle, {dt:.1f} s on {cores} threads"}


# ------------------------------------------------------------- helpers
def dist_env():
    return int(os.environ.get("WORLD_SIZE", "1")), int(os.environ.get("RANK", "0")), \
        int(os.environ.get("LOCAL_RANK", "0"))


def load_peaks():
    try:
        return json.load(open(PEAKS_PATH))
    except Exception:
        return None


def work_flops(w, d):
    """Algorithmic FP32 FLOPs of the update: squared distance to a staged
    cell 2d (d FMA), accumulation of a summary / neighbour 2d (adds), scanned-point distance 3d,
    subtree box test (min+max distance) 6d."""
    return 2 * d * w["cls"] + 2 * d * w["acc"] + 3 * d * w["scan"] + 6 * d * w["node"]


def traffic_from_profiles(name="ncu_update_traffic.json"):
    p = os.path.join(ROOT, "profiles", name)
    try:
        return json.load(open(p)).get("bytes_per_launch")
    except Exception:
        return None


# ------------------------------------------------------------ our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_edbt_jorgensena23_b200 import datagen, distributed as DR, eggsync as E

    world, rank, local = dist_env()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    c = datagen.make_config(args.config)
    X = c.generate(args.seed)
    n, d = X.shape
    # one explicit stream for the library, the L2 flush, the events and the collectives
    # (the legacy default stream has handle 0, which the library would replace by its own)
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)
    Xd = torch.from_numpy(X).to(dev)
    ctx = E.Context(n, d, c.eps, device=local, stream=stream.cuda_stream)
    comm = DR.TorchComm(n, d, dev, ctx=ctx) if world > 1 else DR.LocalComm(n)
    flush = torch.empty(256 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)

    class Hooks:
        def __init__(self):
            self.ev = []

        def before_update(self):
            e = torch.cuda.Event(enable_timing=True)
            e.record(stream)
            self.ev.append([e, None])

        def after_update(self):
            e = torch.cuda.Event(enable_timing=True)
            e.record(stream)
            self.ev[-1][1] = e

    def one_step(hooks=None):
        ctx.load(Xd)
        it, ok, lab = DR.run(ctx, comm, hooks=hooks)
        return it, ok, lab

    for _ in range(args.warmup):
        flush.zero_()
        it, ok, lab = one_step()
    assert ok, "clustering did not converge"
    # instrumented pass (untimed): algorithmic work of the update launches (SIMT kernel
    # counters; the tensor-core kernel's work is counted from its plan, below)
    ctx.work(enable=1)
    one_step()
    work = ctx.work(enable=0)
    ctx.tc_work(enable=1)  # time every tensor-core update launch (CUDA events on the library stream)
    # timed region
    hooks = Hooks()
    step_ms = []
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches0 = ctx.launches()
    with ClockSampler(local) as clk:
        for _ in range(args.steps):
            flush.zero_()
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            it, ok, lab = one_step(hooks)
            e1.record(stream)
            torch.cuda.synchronize()
            step_ms.append(e0.elapsed_time(e1))
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches = ctx.launches() - launches0
    tcw = ctx.tc_work(enable=0)
    upd_ms = [a.elapsed_time(b) for a, b in hooks.ev]
    ms = statistics.mean(step_ms)
    if world > 1:
        t = torch.tensor([ms, sum(upd_ms) / len(upd_ms)], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms, upd_avg = float(t[0]), float(t[1])
    else:
        upd_avg = sum(upd_ms) / len(upd_ms)
    iters = it
    value = n * iters / (ms / 1e3)

    peaks = load_peaks()
    clk_s = clk.summary()
    fmax = (peaks or {}).get("sm_max_mhz") or clk_s["sm_max_mhz"] or 1965.0
    upd_share = sum(upd_ms) / sum(step_ms)
    if tcw["launches"] > 0:
        # roofline of the dominant kernel, k_update_tc: tcgen05 tensor cores.  achieved = the
        # METHOD's FLOPs per launch / the kernel's own event time (CUDA events on the library
        # stream, every launch of the timed region).  Method FLOPs per (point, entry) pair
        # (DESIGN.md §6): the expanded distance |p-c|^2 - lim = -2 q.c' - L, d+2 MACs (GEMM1,
        # kind::f16), plus the masked Eq.5 sums P.[sum sin | sum cos | count], 2d+1 MACs (GEMM2,
        # kind::i8): 2((d+2)+(2d+1)) FLOPs.  The hi/lo fp16 splits and base-256 digit columns
        # that make those products exact are emulation overhead, reported separately
        # (emulated_flops_per_step), not counted as achieved work.
        # peak: each part at its own dtype's peak, fp16 dense = bf16 (measured), int8 dense = 2x
        # bf16 (B200_PROFILING.md nominal 4.5 vs 2.25 PF); the combined peak is the rate at
        # which both parts of a pair would run back to back at those peaks:
        #   P = f_all / (f_dist / P16 + f_sum / P8).
        tc_ns = tcw["ns"] / tcw["launches"]
        pairs_per_launch = tcw["pairs"] / tcw["launches"]
        f_dist, f_sum = 2 * (d + 2), 2 * (2 * d + 1)
        method_flops_per_pair = f_dist + f_sum
        achieved = pairs_per_launch * method_flops_per_pair / (tc_ns * 1e-9) / 1e12
        bf16 = (peaks or {}).get("bf16_tflops_sustained")
        bf16_burst = (peaks or {}).get("bf16_tflops")

        def comb(p16):
            return method_flops_per_pair / (f_dist / p16 + f_sum / (2.0 * p16))

        peak = comb(bf16 if bf16 else 1590.0)
        roof = {"bound": "tensor", "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                "traffic": traffic_from_profiles("ncu_update_tc_traffic.json"),
                "kernel": "k_update_tc (A6 EGG-update on tcgen05: fp16 distance GEMM + exact int8 summary GEMM)",
                "kernel_ms_per_launch": tc_ns / 1e6, "launches_per_step": tcw["launches"] / args.steps,
                "pairs_per_step": tcw["pairs"] / args.steps,
                "method_flops_per_pair": method_flops_per_pair,
                "emulated_flops_per_step": tcw["flops"] / args.steps,
                "frac_vs_burst_peak": (achieved / comb(bf16_burst)) if bf16_burst else None,
                "peak_basis": ("f_dist=2(d+2) at fp16 dense (= MEASURED_PEAKS bf16_tflops_sustained) and "
                               "f_sum=2(2d+1) at int8 dense (2x that, B200_PROFILING.md nominal ratio), combined "
                               "P = (f_dist+f_sum)/(f_dist/P16 + f_sum/P8); sustained because the kernel is timed "
                               "inside a long step" if bf16 else "fallback 1.59 PF bf16, same combination")}
    else:
        # roofline of the dominant kernel (SIMT k_update): FP32 pipe
        flops_per_launch = work_flops(work, d) / iters  # per launch on this rank (its range share)
        achieved = flops_per_launch / (upd_avg / 1e3) / 1e12
        peak = 2 * FP32_LANES * SM_COUNT * fmax * 1e6 / 1e12
        roof = {"bound": "alu", "achieved": achieved, "peak": peak, "unit": "TFLOP/s", "frac": achieved / peak,
                "traffic": traffic_from_profiles(), "kernel": "k_update (A6 EGG-update)",
                "peak_basis": f"FP32 FMA pipe 2*128 lanes*148 SMs*{fmax:.0f} MHz (sm_max_mhz, MEASURED_PEAKS.json)"}

    # end-to-end through the C ABI with pinned host buffers (rank 0 at N=1 only)
    e2e = None
    cpu = None
    if world == 1 and not args.no_e2e:
        pin = torch.empty((n, d), dtype=torch.float32, pin_memory=True)
        pin.numpy()[:] = X
        Xp = pin.numpy()
        lab_pin = torch.empty(n, dtype=torch.int32, pin_memory=True).numpy()
        ts = []
        for k in range(args.warmup + args.steps):
            flush.zero_()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            r = E.cluster(Xp, c.eps)
            dt = time.perf_counter() - t0
            lab_pin[:] = r["labels"]
            if k >= args.warmup:
                ts.append(dt)
        te = statistics.mean(ts)
        e2e = {"value": n * r["iters"] / te, "unit": UNIT, "h2d_bytes_per_step": int(n * d * 4),
               "d2h_bytes_per_step": int(n * 4), "seconds": te,
               "how": "wall time of the synchronous eggsync_cluster() call from pinned host points to host labels "
                      "(workspace alloc/free, H2D, all iterations, D2H)"}
    if world == 1 and not args.no_cpu:
        cpu = cpu_baseline_obj(X, c, args.cpu_seconds)
    # context (not the metric): one direct all-pairs Eq.1 update (GPU-SynC style, F4) of the same
    # D^0 on the same GPU, against the grid path's mean iteration of the timed clusterings
    direct = None
    if world == 1 and not args.no_direct:
        Xd0 = torch.from_numpy(X).cuda()
        tds = []
        for k in range(2):
            u = Xd0.clone()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            E.sync_step(u, c.eps)  # synchronous (reads r_c back)
            if k:
                tds.append((time.perf_counter() - t0) * 1e3)
        direct = {"ms_per_iteration": tds[0], "grid_ms_per_iteration": ms / iters,
                  "grid_speedup": tds[0] / (ms / iters),
                  "how": "wall time of one synchronous eggsync_sync_step on device-resident D^0 (k_sync_brute, "
                         "O(n^2 d), scratch alloc included, 1 warm-up); grid = ms_per_step / iters"}
    if rank != 0:
        return
    line = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "f32",
        "data": "synthetic",
        "config": {"workload": workload_desc(c), "n": n, "d": d, "eps": c.eps, "iters": iters,
                   "clustering_s": ms / 1e3, "clusters": int(lab.max()) + 1,
                   "parallelism": f"replicate + block-interleaved ownership + NCCL all-gather x{world}" if world > 1 else "single GPU",
                   "l2": "flushed between steps (256 MiB write); inputs resident in HBM",
                   "update_share_of_step": upd_share, "update_ms_per_launch": upd_avg,
                   "launches_per_step": launches / args.steps, "work_counters": work},
        "roofline": roof,
        "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": launches, "clocks": clk_s,
        "direct_path_context": direct,
    }
    print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


# ------------------------------------------------- E2: sharded points (C5)
def run_shard(args):
    """--shard: SURVEY.md §8(e) E2 -- no rank holds all points (slab shards + halo exchange,
    distributed.run_sharded); one step = one complete clustering.  Device time (CUDA events
    on the current stream, barrier on both sides), max over ranks."""
    import torch
    import torch.distributed as dist

    from paper_conf_edbt_jorgensena23_b200 import datagen, distributed as DR, eggsync as E

    world, rank, local = dist_env()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    dist.init_process_group("nccl" if world > 1 else "gloo", device_id=dev if world > 1 else None,
                            **({} if world > 1 else {"rank": 0, "world_size": 1,
                                                     "init_method": "tcp://127.0.0.1:%d" % _free_port()}))
    c = datagen.make_config(args.config)
    X = c.generate(args.seed)
    n, d = X.shape
    share = np.array_split(np.arange(n), world)[rank]
    stream = torch.cuda.Stream(dev)
    torch.cuda.set_stream(stream)
    Xd = torch.from_numpy(X[share]).to(dev)
    gd = torch.from_numpy(share.astype(np.int64)).to(dev)
    ex = DR.ShardExchange(d, c.eps, dev)
    make = lambda m, dd: E.Context(m, dd, c.eps, device=local, stream=stream.cuda_stream)  # noqa: E731

    def one():
        return DR.run_sharded(Xd, gd, c.eps, ex, make)

    for _ in range(args.warmup):
        it, ok, lab, _ = one()
    ms = []
    dist.barrier()
    torch.cuda.synchronize()
    with ClockSampler(local) as clk:
        for _ in range(args.steps):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            it, ok, lab, _ = one()
            e1.record(stream)
            torch.cuda.synchronize()
            ms.append(e0.elapsed_time(e1))
    dist.barrier()
    t = torch.tensor([statistics.mean(ms)], dtype=torch.float64, device=dev if world > 1 else "cpu")
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    msv = float(t[0])
    if rank == 0:
        print(json.dumps({
            "metric": METRIC, "value": n * it / (msv / 1e3), "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": msv, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": {"workload": workload_desc(c), "n": n, "d": d, "eps": c.eps, "iters": it, "converged": ok,
                       "clusters": int(lab.max()) + 1, "parallelism": f"E2 sharded points: slab shards + halo x{world}",
                       "l2": "inputs resident in HBM (n*d*4 B per rank share); no flush (whole clusterings)"},
            "clocks": clk.summary(), "gpu_launches": None}), flush=True)
    dist.destroy_process_group()


def _free_port():
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        return sk.getsockname()[1]


# ---------------------------------------------------- reference arm (oracle)
def run_reference(args):
    world, rank, _ = dist_env()
    if rank != 0:
        return
    from paper_conf_edbt_jorgensena23_b200 import datagen
    c = datagen.make_config(args.config)
    X = c.generate(args.seed)
    rate0, m, dt, cores = oracle_rate(X, c.eps, args.cpu_seconds / 2)
    rng = np.random.default_rng(1)
    import oracle
    ts = []
    for k in range(args.warmup + args.steps):
        idx = rng.choice(len(X), m, replace=False)
        t0 = time.perf_counter()
        oracle.step_sample(X, c.eps, idx)
        if k >= args.warmup:
            ts.append(time.perf_counter() - t0)
    sec = statistics.mean(ts)
    value = m / sec
    sample = (f"{m} Eq.1 point-updates per step of {c.name} iteration 1 (each against the full n={c.n:,} state), "
              f"fp64 C/OpenMP oracle on {cores} threads")
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": sec * 1e3, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": workload_desc(c), "n": c.n, "d": c.d, "eps": c.eps, "sample_points_per_step": m},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def relaunch(n: int):
    """--gpus N without a launcher: start N ranks with torch.distributed.run on this node
    (127.0.0.1 rendezvous), or fail loudly when the node has fewer than N GPUs."""
    import torch
    have = torch.cuda.device_count()
    if have < n:
        sys.exit(f"bench.py: --gpus {n} requested but this node has {have} CUDA device(s)")
    import socket
    with socket.socket() as sk:
        sk.bind(("127.0.0.1", 0))
        port = sk.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr=127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
    os.execv(sys.executable, cmd)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", choices=["ours", "reference"], default="ours")
    ap.add_argument("--config", default="C3")
    ap.add_argument("--seed", type=int, default=0)
    ap.add_argument("--cpu-seconds", type=float, default=12.0)
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-direct", action="store_true", help="skip the direct-path (GPU-SynC-style) context timing")
    ap.add_argument("--shard", action="store_true", help="E2: sharded points (slab shards + halo), e.g. --config C5")
    args = ap.parse_args()
    if args.warmup < 3:
        args.warmup = 3
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        relaunch(args.gpus)  # one rank per GPU under torch.distributed.run (never returns)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus:
        sys.exit(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}; launch one rank per GPU")
    if args.impl == "reference":
        run_reference(args)
    elif args.shard:
        run_shard(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
