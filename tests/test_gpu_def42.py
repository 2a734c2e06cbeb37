"""GPU parity of term_mode = EGGSYNC_TERM_DEF42: Def 4.2 literally (L106-110)
on the grid structure (csrc/def42_grid.cu) and, as EGGSYNC_TERM_DEF42_DIRECT, on the direct
all-pairs kernels (csrc/sync_brute.cu); each against oracle_cluster's DEF42 mode:
identical labels (eps-components of the returned state, canonical), equal iteration counts,
coordinates within 1e-4.  The partition equals the grid mode's (Theorem 4.7) and DEF42 never
needs more iterations (the grid first term implies Def 4.2 term (i): cell diagonal eps/2, L252).
"""
import numpy as np
import pytest

import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen
from paper_conf_edbt_jorgensena23_b200 import eggsync as E

pytestmark = pytest.mark.gpu


MODES = [E.TERM_DEF42, E.TERM_DEF42_DIRECT]


def _check(X, eps, max_iters=10000, mode=E.TERM_DEF42):
    g = E.cluster(X, eps, coords=True, term_mode=mode, max_iters=max_iters)
    o = oracle.cluster(X, eps, term_mode=oracle.DEF42, max_iters=max_iters)
    assert o["rc"] in (oracle.OK, oracle.NOT_CONVERGED)
    assert g["converged"] == (o["rc"] == oracle.OK)
    assert g["iters"] == o["iters"]
    assert np.array_equal(g["labels"], o["labels"])
    assert np.abs(g["coords"].astype(np.float64) - o["X"]).max() <= 1e-4
    return g


@pytest.mark.parametrize("mode", MODES)
@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_def42_c1_matches_oracle_and_grid(seed, mode):
    X = datagen.blobs(1000, 2, 5, seed=seed)
    g = _check(X, 0.05, mode=mode)
    grid = E.cluster(X, 0.05)
    assert np.array_equal(g["labels"], grid["labels"]) and g["iters"] <= grid["iters"]


@pytest.mark.parametrize("n,d,k,eps,noise", [(2000, 5, 10, 0.05, 0.0), (2000, 10, 20, 0.1, 0.05),
                                             (1500, 3, 4, 0.05, 0.1), (700, 1, 3, 0.02, 0.0),
                                             (400, 32, 4, 0.3, 0.0)])
@pytest.mark.parametrize("mode", MODES)
def test_def42_dims_match_oracle(n, d, k, eps, noise, mode):
    _check(datagen.blobs(n, d, k, noise=noise, seed=5), eps, mode=mode)


@pytest.mark.parametrize("mode", MODES)
def test_def42_bridge_and_max_iters(mode):
    X = datagen.bridge()
    _check(X, 0.05, mode=mode)
    g = _check(X, 0.05, max_iters=3, mode=mode)  # not converged: labels = eps-components of the last state
    assert not g["converged"] and g["iters"] == 3


@pytest.mark.parametrize("mode", MODES)
def test_def42_edge_cases(mode):
    _check(np.array([[0.25, 0.75]], np.float32), 0.05, mode=mode)              # n = 1
    _check(np.repeat(datagen.uniform(30, 3, seed=2), 4, axis=0), 0.05, mode=mode)  # exact duplicates
    _check(datagen.uniform(500, 2, seed=3), 0.9, mode=mode)                    # eps covers everything


@pytest.mark.parametrize("cfg", ["C2", "C4-d5", "C4-d10"])
def test_def42_grid_equals_direct_at_full_size(cfg):
    """Two independent GPU implementations of Def 4.2 (grid traversal vs all pairs) at BASELINE
    sizes: identical labels and iterations, coordinates equal (the same grid update runs in both:
    the direct mode's update is Eq.1 over all pairs, so within 2e-6 per step)."""
    c = datagen.make_config(cfg)
    X = c.generate(0)
    g = E.cluster(X, c.eps, coords=True, term_mode=E.TERM_DEF42)
    h = E.cluster(X, c.eps, coords=True, term_mode=E.TERM_DEF42_DIRECT)
    assert g["converged"] and h["converged"]
    assert g["iters"] == h["iters"]
    assert np.array_equal(g["labels"], h["labels"])
    assert np.abs(g["coords"] - h["coords"]).max() <= 1e-4
    grid = E.cluster(X, c.eps)
    assert np.array_equal(g["labels"], grid["labels"]) and g["iters"] <= grid["iters"]


@pytest.mark.parametrize("mode", MODES)
def test_def42_device_pointers_and_domain(mode):
    import torch
    X = datagen.blobs(1000, 2, 5, seed=6)
    h = E.cluster(X, 0.05, term_mode=mode)
    t = E.cluster(torch.from_numpy(X).cuda(), 0.05, term_mode=mode)
    assert np.array_equal(t["labels"].cpu().numpy(), h["labels"]) and t["iters"] == h["iters"]
    bad = X.copy()
    bad[7, 1] = 1.5
    with pytest.raises(E.EggSyncError) as ei:
        E.cluster(bad, 0.05, term_mode=mode)
    assert ei.value.rc == E.EDOMAIN
