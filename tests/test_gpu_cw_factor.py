"""GPU parity with a grid cell width below the L252 bound (opts.cw_factor).

c_w = f * eps / (2 sqrt d), f in (0, 1].  Same bars as test_gpu_parity.py against the oracle
run with the same f: identical labels and iteration counts, coordinates within 1e-4 at the end,
identical neighbour counts and criterion flags per step.  At full C2 size (no oracle): the
partition equals the f = 1 partition (Theorem 4.7).
"""
import numpy as np
import pytest

import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen
from paper_conf_edbt_jorgensena23_b200 import eggsync as E

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("f", [0.5, 0.3])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_cluster_c1_matches_oracle(f, seed):
    X = datagen.blobs(1000, 2, 5, seed=seed)
    g = E.cluster(X, 0.05, coords=True, cw_factor=f)
    o = oracle.cluster(X, 0.05, cw_factor=f)
    assert o["rc"] == oracle.OK and g["converged"]
    assert g["iters"] == o["iters"]
    assert np.array_equal(g["labels"], o["labels"])
    assert np.abs(g["coords"].astype(np.float64) - o["X"]).max() <= 1e-4


@pytest.mark.parametrize("n,d,k,eps,f", [(3000, 10, 20, 0.1, 0.5), (2000, 5, 10, 0.05, 0.7), (1500, 3, 4, 0.05, 0.25)])
def test_cluster_higher_d_matches_oracle(n, d, k, eps, f):
    X = datagen.blobs(n, d, k, seed=3)
    g = E.cluster(X, eps, coords=True, cw_factor=f)
    o = oracle.cluster(X, eps, cw_factor=f)
    assert o["rc"] == oracle.OK and g["converged"]
    assert g["iters"] == o["iters"]
    assert np.array_equal(g["labels"], o["labels"])
    assert np.abs(g["coords"].astype(np.float64) - o["X"]).max() <= 1e-4


def test_step_flags_match_oracle():
    """Step through a C1 run with f = 0.5: counts, coordinates and both criterion terms agree."""
    X = datagen.blobs(1000, 2, 5, seed=4)
    for _ in range(12):
        g = E.step(X, 0.05, nbr=True, cw_factor=0.5)
        Xo, nbr, fl = oracle.step(X, 0.05, compute_f2=True, cw_factor=0.5)
        assert np.array_equal(g["nbr"], nbr)
        assert np.abs(g["points"].astype(np.float64) - Xo).max() <= 2e-6
        assert g["first"] == fl[0]
        assert g["second"] == (fl[2] if fl[0] == 1 else -1)
        if g["synced"]:
            break
        X = g["points"]
    assert g["synced"] == 1


def test_c2_partition_independent_of_cell_width():
    c = datagen.make_config("C2")
    X = datagen.blobs(c.n, c.d, c.k, noise=c.noise, seed=0)
    a = E.cluster(X, c.eps)
    b = E.cluster(X, c.eps, cw_factor=0.5)
    assert a["converged"] and b["converged"] and b["iters"] >= a["iters"]
    assert np.array_equal(a["labels"], b["labels"])
