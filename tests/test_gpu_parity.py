"""GPU parity: the CUDA path (through the C ABI) against the fp64 oracle.

Bars:
  * integer neighbour counts |N_eps(p)| identical (the eps-predicate is decided
    in fp64 exactly as the oracle inside the fp32 error band);
  * one-step coordinates within 2e-6 of the fp64 oracle on the same fp32 input;
  * full clustering: identical canonical labels, equal iteration count,
    final coordinates within 1e-4 (north_star);
  * first / second term flags identical.
"""
import json
import os

import numpy as np
import pytest

import oracle
from tests import theorem47
from paper_conf_edbt_jorgensena23_b200 import datagen
from paper_conf_edbt_jorgensena23_b200 import eggsync as E

pytestmark = pytest.mark.gpu
GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "worked_examples.json")))


def _step_compare(X, eps, atol=2e-6):
    g = E.step(X, eps, nbr=True)
    Xo, nbr_o, f = oracle.step(X, eps)
    assert np.array_equal(g["nbr"], nbr_o), f"neighbour counts differ at {np.nonzero(g['nbr'] != nbr_o)[0][:10]}"
    err = np.abs(g["points"].astype(np.float64) - Xo).max()
    assert err <= atol, err
    assert g["first"] == f[0]
    if f[0] == 1:
        _, _, f2 = oracle.step(X, eps, compute_f2=True)
        assert g["second"] == f2[2]
    else:
        assert g["second"] == -1
    return g


@pytest.mark.parametrize("seed", [0, 1, 2])
@pytest.mark.parametrize("n,d,k,eps", [(1000, 2, 5, 0.05), (3000, 3, 4, 0.08), (2500, 5, 6, 0.1),
                                       (4000, 10, 5, 0.2), (777, 7, 3, 0.15), (1500, 1, 3, 0.02),
                                       (2000, 12, 4, 0.25), (1800, 11, 3, 0.25)])
def test_step_parity(seed, n, d, k, eps):
    _step_compare(datagen.blobs(n, d, k, seed=seed), eps)


@pytest.mark.parametrize("seed", [0, 1])
def test_step_parity_uniform_and_noise(seed):
    _step_compare(datagen.uniform(3000, 3, seed=seed), 0.06)
    _step_compare(datagen.blobs(3000, 4, 5, noise=0.2, seed=seed), 0.1)


def test_step_parity_iterated_states():
    """Later iterations: dense cells, full-cell and full-subtree fast paths."""
    X = datagen.blobs(3000, 3, 4, seed=4)
    for _ in range(4):
        g = _step_compare(X, 0.08)
        X = g["points"]


def test_step_parity_big_cells():
    """Many points in few cells (cells spanning warps; partial-cell scans of large cells)."""
    rng = np.random.default_rng(0)
    base = rng.random((6, 3)).astype(np.float32)
    X = (base[rng.integers(0, 6, 5000)] + rng.normal(0, 0.002, (5000, 3))).astype(np.float32)
    X = np.clip(X, 0, 1)
    _step_compare(X, 0.05)
    _step_compare(X, 0.006)


def test_step_boundary_pairs():
    """Pairs at exactly eps and one ulp beyond: the fp64 band decides them like the oracle."""
    e = np.float32(0.05)
    X = np.array([[0.0, 0.5], [e, 0.5], [0.3, 0.3], [0.3 + np.nextafter(e, np.float32(1)), 0.3],
                  [1.0, 1.0], [1.0 - e, 1.0]], np.float32)
    g = _step_compare(X, float(e))
    # 1.0 - fl32(1 - e) = 0.0500000119 > e: the last pair is NOT within eps (fp32 input rounding)
    assert g["nbr"].tolist() == [2, 2, 1, 1, 1, 1]


@pytest.mark.parametrize("name", [k for k in GOLD if not k.startswith("_")])
def test_worked_examples_gpu(name):
    g = GOLD[name]
    r = E.cluster(np.array(g["points"], np.float32), g["eps"])
    assert r["converged"]
    assert r["iters"] == g["iters"], g["cite"]
    assert r["labels"].tolist() == g["labels"], g["cite"]


def _cluster_compare(X, eps, coord_tol=1e-4):
    g = E.cluster(X, eps, coords=True)
    o = oracle.cluster(X, eps)
    assert o["rc"] == oracle.OK and g["converged"]
    assert np.array_equal(g["labels"], o["labels"])
    assert g["iters"] == o["iters"]
    assert np.abs(g["coords"].astype(np.float64) - o["X"]).max() <= coord_tol
    return g, o


@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_cluster_parity_c1(seed):
    """BASELINE config C1: 2-D blobs n=1000, 5 clusters, eps=0.05."""
    c = datagen.CONFIGS["C1"]
    _cluster_compare(c.generate(seed), c.eps)


@pytest.mark.parametrize("n,d,k,noise,eps,seed", [(4000, 3, 5, 0.0, 0.05, 0), (3000, 5, 10, 0.0, 0.05, 1),
                                                  (5000, 10, 20, 0.05, 0.1, 0), (2000, 20, 5, 0.0, 0.05, 2),
                                                  (3333, 4, 3, 0.1, 0.07, 5), (1024, 32, 4, 0.0, 0.4, 1),
                                                  # d=32 at 6 key bits per dimension: 4 update warps
                                                  # would need 234 KB of shared memory (UpdWarps)
                                                  (1500, 32, 4, 0.0, 0.3, 2), (1200, 29, 3, 0.05, 0.2, 3)])
def test_cluster_parity_shapes(n, d, k, noise, eps, seed):
    _cluster_compare(datagen.blobs(n, d, k, noise=noise, seed=seed), eps)


@pytest.mark.parametrize("pts,eps,iters,labels", [
    ([[0.25, 0.75]], 0.05, 1, [0]),
    ([[0.3, 0.3]] * 70, 0.05, 1, [0] * 70),
    ([[0.0, 0.0], [1.0, 1.0], [0.0, 1.0], [1.0, 0.0]], 0.05, 1, [0, 1, 2, 3]),
])
def test_edge_cases(pts, eps, iters, labels):
    r = E.cluster(np.array(pts, np.float32), eps)
    assert r["iters"] == iters and r["labels"].tolist() == labels


def test_domain_error_leaves_outputs():
    X = np.array([[0.5, 0.5], [0.5, 1.5]], np.float32)
    with pytest.raises(E.EggSyncError) as ei:
        E.cluster(X, 0.05)
    assert ei.value.rc == E.EDOMAIN
    X[1, 1] = np.nan
    with pytest.raises(E.EggSyncError):
        E.step(X, 0.05)


def test_eps_covers_everything():
    X = datagen.uniform(500, 2, seed=3)
    _cluster_compare(X, 1.5)


def test_max_iters_not_converged():
    X = np.array([[0.40, 0.5], [0.44, 0.5], [0.48, 0.5]], np.float32)
    r = E.cluster(X, 0.05, max_iters=1)
    assert not r["converged"] and r["iters"] == 1


def test_determinism():
    X = datagen.blobs(20000, 5, 8, noise=0.05, seed=7)
    a = E.cluster(X, 0.08, coords=True)
    b = E.cluster(X, 0.08, coords=True)
    assert np.array_equal(a["labels"], b["labels"]) and a["iters"] == b["iters"]
    assert np.array_equal(a["coords"], b["coords"])


def test_device_pointer_path_matches_host():
    import torch
    X = datagen.blobs(5000, 3, 5, seed=1)
    h = E.cluster(X, 0.05, coords=True)
    t = torch.from_numpy(X).cuda()
    dv = E.cluster(t, 0.05, coords=True)
    torch.cuda.synchronize()
    assert np.array_equal(dv["labels"].cpu().numpy(), h["labels"])
    assert np.array_equal(dv["coords"].cpu().numpy(), h["coords"])


def test_context_phases_match_cluster():
    X = datagen.blobs(6000, 4, 5, seed=2)
    ref = E.cluster(X, 0.07, coords=True)
    ctx = E.Context(len(X), 4, 0.07)
    ctx.load(X)
    it, ok = ctx.run()
    assert ok and it == ref["iters"]
    assert np.array_equal(ctx.labels(), ref["labels"])
    assert np.array_equal(ctx.coords(), ref["coords"])


# ------------------------------------------------------------ full-size (C3)
@pytest.fixture(scope="module")
def c3():
    c = datagen.CONFIGS["C3"]
    return c, c.generate(0)


def test_c3_first_step_sampled(c3):
    """BASELINE config C3 at full size (n=1M, d=10): the update of sampled points equals the
    oracle's per-point definition; neighbour counts identical."""
    c, X = c3
    g = E.step(X, c.eps, nbr=True)
    idx = np.random.default_rng(0).choice(len(X), 192, replace=False)
    Xs, ns = oracle.step_sample(X, c.eps, idx)
    assert np.array_equal(g["nbr"][idx], ns)
    assert np.abs(g["points"][idx].astype(np.float64) - Xs).max() <= 2e-6


def test_c3_cluster_terminal_property(c3):
    """C3 full clustering: Theorem 4.7 on the final state for sampled points
    (same label <=> within eps), labels canonical, converged."""
    c, X = c3
    r = E.cluster(X, c.eps, coords=True)
    assert r["converged"]
    lab = r["labels"]
    first = np.unique(lab, return_index=True)[1]
    assert np.array_equal(np.sort(first), first)  # canonical: ids by first occurrence
    idx = np.random.default_rng(1).choice(len(X), 64, replace=False)
    assert oracle.terminal_violations(r["coords"], c.eps, lab, idx) == 0
    # the complete Theorem 4.7 property over all n (tests/theorem47.py: independent of the
    # CUDA path and of the oracle): same label <=> within eps, for every pair
    assert theorem47.violations(r["coords"], lab, c.eps) == 0
    # Def 4.2 evaluated literally (term_mode DEF42, another criterion and another labelling:
    # eps-graph components) reaches the same partition (Theorem 4.7), in no more iterations
    d42 = E.cluster(X, c.eps, term_mode=E.TERM_DEF42)
    assert d42["converged"] and np.array_equal(d42["labels"], lab) and d42["iters"] <= r["iters"]


# ------------------------------------------------------------ full-size (C5, one GPU)
@pytest.fixture(scope="module")
def c5():
    c = datagen.CONFIGS["C5"]
    return c, c.generate(0)


def test_c5_first_step_sampled(c5):
    """BASELINE config C5 at full size on one GPU (n=10M, d=3: ~564k neighbours per point,
    2.5e10 plan entries, so the update falls back from the tensor-core slot lists to the SIMT
    kernel): sampled point updates and neighbour counts equal the oracle's definition."""
    c, X = c5
    g = E.step(X, c.eps, nbr=True)
    idx = np.random.default_rng(0).choice(len(X), 48, replace=False)
    Xs, ns = oracle.step_sample(X, c.eps, idx)
    assert np.array_equal(g["nbr"][idx], ns)
    assert np.abs(g["points"][idx].astype(np.float64) - Xs).max() <= 2e-6


def test_c5_cluster_terminal_property(c5):
    c, X = c5
    r = E.cluster(X, c.eps, coords=True)
    assert r["converged"]
    idx = np.random.default_rng(1).choice(len(X), 32, replace=False)
    assert oracle.terminal_violations(r["coords"], c.eps, r["labels"], idx) == 0


def test_pack_unpack_roundtrip_multi_rank_layout():
    """The all-gather plumbing kernels: packing 3 rank ranges of D^{t+1} and unpacking the
    concatenated (ranks*d, cnt) buffer reproduces the next state exactly (bitwise, ragged tail)."""
    import torch
    from paper_conf_edbt_jorgensena23_b200 import distributed as DR
    X = datagen.blobs(1001, 3, 4, seed=3)
    ref = E.Context(len(X), 3, 0.07)
    ref.load(X)
    it_ref, ok_ref, lab_ref = DR.run(ref)

    class FakeComm:  # 3 "ranks" emulated in one process: every range is updated and exchanged
        world, cnt = 3, (1001 + 2) // 3

        def __init__(self):
            self.lo, self.hi = 0, 1001

        def reduce_min(self, v):
            return v

        def update(self, ctx):
            ctx.update(self.lo, self.hi)

        def exchange(self, ctx):
            parts = [torch.empty((3, self.cnt), device="cuda") for _ in range(3)]
            for r in range(3):
                ctx.pack_into(r * self.cnt, self.cnt, parts[r])
            g = torch.cat(parts, 0)
            ctx.unpack_from(g.view(3, -1, self.cnt), 3, self.cnt)

    ctx = E.Context(len(X), 3, 0.07)
    ctx.load(X)
    it, ok, lab = DR.run(ctx, FakeComm())
    assert ok and ok_ref and it == it_ref
    assert np.array_equal(lab, lab_ref)
    assert np.array_equal(ctx.coords(), ref.coords())

    class FakeOwned(FakeComm):  # block-interleaved ownership, 3 emulated ranks
        def update(self, ctx):
            for r in range(3):
                ctx.update_owned(r, 3)

        def exchange(self, ctx):
            cnt = ctx.owned_count(3)
            parts = [torch.empty((3, cnt), device="cuda") for _ in range(3)]
            for r in range(3):
                ctx.pack_owned_into(r, 3, parts[r])
            ctx.unpack_owned_from(torch.cat(parts, 0).view(3, -1, cnt), 3)

    ctx2 = E.Context(len(X), 3, 0.07)
    ctx2.load(X)
    it2, ok2, lab2 = DR.run(ctx2, FakeOwned())
    assert ok2 and it2 == it_ref and np.array_equal(lab2, lab_ref)
    assert np.array_equal(ctx2.coords(), ref.coords())


def test_nccl_single_rank_driver():
    """torch.distributed NCCL process group of size 1 through TorchComm equals the local run."""
    import torch
    import torch.distributed as dist
    from paper_conf_edbt_jorgensena23_b200 import distributed as DR
    X = datagen.blobs(3000, 4, 5, seed=1)
    ref = E.cluster(X, 0.07)
    os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
    os.environ.setdefault("MASTER_PORT", "29533")
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        s = torch.cuda.Stream()
        torch.cuda.set_stream(s)
        ctx = E.Context(len(X), 4, 0.07, device=0, stream=s.cuda_stream)
        ctx.load(X)
        it, ok, lab = DR.run(ctx, DR.TorchComm(len(X), 4, torch.device("cuda", 0), ctx=ctx))
        assert ok and it == ref["iters"] and np.array_equal(lab, ref["labels"])
    finally:
        dist.destroy_process_group()
        torch.cuda.set_stream(torch.cuda.default_stream())


# ------------------------------------------------- BASELINE configs C2 / C4
def test_c2_full_oracle_parity():
    """BASELINE config C2 (n=70,000, d=5, 10 clusters, eps=0.05) against the full O(T n^2 d)
    oracle: identical labels, equal iteration count, coordinates within 1e-4 (~1 min of host CPU)."""
    c = datagen.CONFIGS["C2"]
    g, o = _cluster_compare(c.generate(0), c.eps)
    assert g["iters"] == 7 and int(g["labels"].max()) + 1 == 24


@pytest.mark.parametrize("d", [2, 5, 10, 15, 20])
def test_c4_dimension_sweep_sampled(d):
    """BASELINE config C4 (n=100,000, d=2..20, eps=0.05) at full size: the first update of
    sampled points and their neighbour counts equal the oracle's per-point definition, and
    the final clustering satisfies Theorem 4.7 for sampled points against all n."""
    c = datagen.make_config(f"C4-d{d}")
    X = c.generate(0)
    g = E.step(X, c.eps, nbr=True)
    idx = np.random.default_rng(d).choice(len(X), 256, replace=False)
    Xs, ns = oracle.step_sample(X, c.eps, idx)
    assert np.array_equal(g["nbr"][idx], ns)
    assert np.abs(g["points"][idx].astype(np.float64) - Xs).max() <= 2e-6
    r = E.cluster(X, c.eps, coords=True)
    assert r["converged"]
    assert oracle.terminal_violations(r["coords"], c.eps, r["labels"], idx[:64]) == 0
