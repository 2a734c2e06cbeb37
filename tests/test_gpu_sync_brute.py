"""GPU parity of the direct SynC path (csrc/sync_brute.cu) through the C ABI.

eggsync_sync_step computes Eq.1 (L68) without the grid and Eq.2's r_c (L74) of the
input state; eggsync_sync_lambda runs Algorithm 1 (L46-56).  Bars:
  * |N_eps(p)| identical to the fp64 oracle (exact fp64 re-decision inside the band);
  * one-step coordinates within 2e-6 of the oracle (fp32 sinf terms, fp64 cross-tile sums);
  * r_c within 1e-6 of the oracle (fp32 expf terms);
  * the grid path (eggsync_step) and the direct path agree: same counts, coordinates within 2e-6;
  * Fig 1 (L89): lambda-termination stops at the oracle's iteration on a state the exact
    criterion rejects, while eggsync_cluster finds the oracle's single cluster.
"""
import numpy as np
import pytest

import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen
from paper_conf_edbt_jorgensena23_b200 import eggsync as E

pytestmark = pytest.mark.gpu


def _compare(X, eps, atol=2e-6):
    g = E.sync_step(X, eps, nbr=True)
    Xo, nbr_o, _ = oracle.step(X, eps)
    r_o, _ = oracle.order_parameter(X, eps)
    assert np.array_equal(g["nbr"], nbr_o), np.nonzero(g["nbr"] != nbr_o)[0][:10]
    err = np.abs(g["points"].astype(np.float64) - Xo).max()
    assert err <= atol, err
    assert abs(g["rc"] - r_o) <= 1e-6, (g["rc"], r_o)
    return g


@pytest.mark.parametrize("n,d,k,eps,seed", [
    (1000, 2, 5, 0.05, 0),     # C1
    (1000, 2, 5, 0.05, 1),
    (3001, 5, 10, 0.05, 2),    # ragged last tile (3001 = 23*128 + 57)
    (2500, 10, 20, 0.1, 3),    # C3-shaped
    (700, 1, 3, 0.02, 4),
    (513, 32, 4, 0.3, 5),      # largest D instantiation
    (1, 3, 1, 0.05, 6),        # single point: never moves, r_c = 1
])
def test_sync_step_matches_oracle(n, d, k, eps, seed):
    X = datagen.blobs(n, d, k, seed=seed)
    g = _compare(X, eps)
    if n == 1:
        assert g["rc"] == 1.0 and np.array_equal(g["points"], X)


def test_sync_step_uniform_and_coincident():
    _compare(datagen.uniform(2000, 3, seed=7), 0.07)
    X = np.repeat(datagen.uniform(40, 4, seed=8), 6, axis=0)  # every point has 5 exact duplicates
    g = _compare(X, 0.05)
    assert (g["nbr"] >= 6).all()


def test_sync_step_device_tensor_in_place():
    import torch
    X = datagen.blobs(5000, 5, 10, seed=9)
    t = torch.from_numpy(X).cuda()
    g = E.sync_step(t, 0.05, nbr=True)
    assert g["points"] is t
    h = E.sync_step(X, 0.05, nbr=True)
    assert np.array_equal(t.cpu().numpy(), h["points"])  # same kernel, same arithmetic
    assert np.array_equal(g["nbr"].cpu().numpy(), h["nbr"]) and g["rc"] == h["rc"]


@pytest.mark.parametrize("cfg", ["C1", "C2"])
def test_grid_path_agrees_with_direct_path(cfg):
    """Two independent GPU implementations of Eq.1 (grid + Eq.5 identity vs direct) on the
    same input, C2 at full size (n=70,000, d=5): identical counts, coordinates within 2e-6."""
    c = datagen.make_config(cfg)
    X = datagen.blobs(c.n, c.d, c.k, noise=c.noise, seed=0)
    g = E.step(X, c.eps, nbr=True)
    b = E.sync_step(X, c.eps, nbr=True)
    assert np.array_equal(g["nbr"], b["nbr"])
    assert np.abs(g["points"].astype(np.float64) - b["points"]).max() <= 2e-6


def test_lambda_termination_fig1():
    X = datagen.bridge()
    g = E.sync_lambda(X, 0.05, 0.999)
    # the oracle's Alg 1 on the same input (state rounded to fp32 after every update, as on the GPU)
    cur, t, r = X.copy(), 0, 0.0
    while r < 0.999:
        r, _ = oracle.order_parameter(cur, 0.05)
        Xn, _, _ = oracle.step(cur, 0.05)
        cur, t = Xn.astype(np.float32), t + 1
    assert g["reached"] and g["iters"] == t == 2
    assert abs(g["rc"] - r) <= 1e-6
    assert np.abs(g["points"].astype(np.float64) - cur).max() <= 2e-6
    s = E.step(g["points"], 0.05)
    assert s["synced"] == 0 and s["first"] == 0  # lambda stopped before the exact criterion holds
    res = E.cluster(X, 0.05)
    o = oracle.cluster(X, 0.05)
    assert res["converged"] and res["iters"] == o["iters"] > t
    assert np.array_equal(res["labels"], o["labels"]) and len(set(res["labels"].tolist())) == 1


def test_lambda_max_iters():
    X = datagen.bridge()
    g = E.sync_lambda(X, 0.05, 1.5, max_iters=3)  # r_c <= 1 < lambda: runs to max_iters
    assert not g["reached"] and g["iters"] == 3


def test_sync_step_c3_full_size_sampled():
    """C3 at full size (n = 1,000,000, d = 10): 96 sampled point updates and r_c terms of the
    direct path against the oracle's per-point definition (oracle_step_sample)."""
    c = datagen.make_config("C3")
    X = datagen.blobs(c.n, c.d, c.k, noise=c.noise, seed=0)
    g = E.sync_step(X, c.eps, nbr=True)
    idx = np.random.default_rng(11).choice(c.n, 96, replace=False)
    Xo, nbr_o = oracle.step_sample(X, c.eps, idx)
    assert np.array_equal(g["nbr"][idx], nbr_o)
    assert np.abs(g["points"][idx].astype(np.float64) - Xo).max() <= 2e-6
    assert 0.0 < g["rc"] < 1.0


@pytest.mark.parametrize("seed", [0, 1])
def test_lambda_loop_c1_matches_oracle(seed):
    X = datagen.blobs(1000, 2, 5, seed=seed)
    g = E.sync_lambda(X, 0.05, 0.999)
    cur, t, r = X.copy(), 0, 0.0
    while r < 0.999:
        r, _ = oracle.order_parameter(cur, 0.05)
        Xn, _, _ = oracle.step(cur, 0.05)
        cur, t = Xn.astype(np.float32), t + 1
    assert g["reached"] and g["iters"] == t and abs(g["rc"] - r) <= 1e-6
    assert np.abs(g["points"].astype(np.float64) - cur).max() <= 1e-5
