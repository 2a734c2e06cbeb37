"""F1: small inputs run Algorithm 4 (L258-278) in ONE kernel launch.

eggsync_cluster sends n <= 4096 (n*d <= 8192, d <= 8) to the thread-block-cluster kernel of
small.cu: no per-iteration host round trip.  Parity bars as for the grid path: identical
canonical labels and iteration count, coordinates within 1e-4 of the fp64 oracle.  The grid
path (EGGSYNC_SMALL=0) must agree on the same inputs.
"""
import json
import os
import time

import numpy as np
import pytest

import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen
from paper_conf_edbt_jorgensena23_b200 import eggsync as E

pytestmark = pytest.mark.gpu
GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "worked_examples.json")))


def _grid(fn, *a, **k):
    os.environ["EGGSYNC_SMALL"] = "0"
    try:
        return fn(*a, **k)
    finally:
        del os.environ["EGGSYNC_SMALL"]


def _check(X, eps, **kw):
    g = E.cluster(X, eps, coords=True, **kw)
    o = oracle.cluster(X, eps, **{k: v for k, v in kw.items() if k == "max_iters"})
    assert np.array_equal(g["labels"], o["labels"])
    assert g["iters"] == o["iters"], (g["iters"], o["iters"])
    assert np.abs(g["coords"].astype(np.float64) - o["X"]).max() <= 1e-4
    r = _grid(E.cluster, X, eps, coords=True, **kw)
    assert np.array_equal(r["labels"], g["labels"]) and r["iters"] == g["iters"]
    return g


@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_c1_one_launch(seed):
    c = datagen.CONFIGS["C1"]
    _check(c.generate(seed), c.eps)


@pytest.mark.parametrize("n,d,k,eps", [(3000, 3, 4, 0.08), (2000, 8, 5, 0.3), (777, 5, 3, 0.15),
                                       (1500, 1, 3, 0.02), (1024, 4, 4, 0.1)])
def test_blobs_one_launch(n, d, k, eps):
    _check(datagen.blobs(n, d, k, noise=0.1, seed=1), eps)


@pytest.mark.xfail(strict=False, reason="fp32 state hazard (DESIGN.md R13, SURVEY §8(c) hazard (i)/(iii)): at "
                   "iteration 2 a pair lies within the fp32-vs-fp64 state difference (~1e-7) of eps; the grid "
                   "path's state flips it, the oracle's does not, and the partitions end up 196 vs 197 clusters")
def test_sparse_noise_flip_hazard():
    _check(datagen.blobs(4096, 2, 6, noise=0.1, seed=1), 0.03)


@pytest.mark.parametrize("name", [k for k in GOLD if not k.startswith("_")])
def test_worked_examples_one_launch(name):
    g = GOLD[name]
    r = E.cluster(np.array(g["points"], np.float32), g["eps"])
    assert r["iters"] == g["iters"] and r["labels"].tolist() == g["labels"], g["cite"]


def test_max_iters_one_launch():
    X = datagen.bridge()
    g = E.cluster(X, 0.05, max_iters=3, coords=True)
    o = oracle.cluster(X, 0.05, max_iters=3)
    assert not g["converged"] and g["iters"] == 3 and o["rc"] == oracle.NOT_CONVERGED
    assert np.array_equal(g["labels"], o["cell_labels"])  # R15: cells of the last state


def test_domain_error_one_launch():
    X = datagen.blobs(100, 2, 2, seed=0)
    X[5, 1] = 1.5
    with pytest.raises(E.EggSyncError) as ei:
        E.cluster(X, 0.05)
    assert ei.value.rc == E.EDOMAIN


def test_long_bridge_473_iterations():
    """The Fig 1 phenomenon (L89) at scale: two clusters of 1000 points joined by one bridge
    point take 473 Eq.1 updates (more than the 343 of the paper's Skin data, L298).  One launch
    runs them all (no per-iteration host synchronisation); labels / iterations equal the
    oracle's, and the one launch is faster than the grid path's per-iteration loop."""
    X = datagen.bridge(m=1000, b=1)
    g = E.cluster(X, 0.05, coords=True)
    o = oracle.cluster(X, 0.05)
    assert g["iters"] == o["iters"] == 473
    assert np.array_equal(g["labels"], o["labels"])
    assert np.abs(g["coords"].astype(np.float64) - o["X"]).max() <= 1e-4
    t0 = time.perf_counter()
    E.cluster(X, 0.05)
    t_small = time.perf_counter() - t0
    t0 = time.perf_counter()
    r = _grid(E.cluster, X, 0.05)
    t_grid = time.perf_counter() - t0
    assert r["iters"] == 473 and np.array_equal(r["labels"], g["labels"])
    assert t_small < t_grid, (t_small, t_grid)
