"""CPU pins of the complete Theorem 4.7 checker (tests/theorem47.py) against brute force."""
import numpy as np
import pytest

import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen
from tests import theorem47


def _brute(X, lab, eps):
    X = X.astype(np.float64)
    e2 = float(np.float32(eps)) ** 2
    t = X[:, None, :] - X[None, :, :]
    near = (t * t).sum(-1) <= e2
    same = lab[:, None] == lab[None, :]
    return int((near != same).sum()) // 2


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_checker_equals_brute_force_on_final_states(seed):
    """On converged oracle states (Theorem 4.7 holds) both counts are 0; on relabelled
    states (two clusters merged, one cluster split) both count the same violating pairs."""
    X = datagen.blobs(400, 3, 4, noise=0.1, seed=seed)
    r = oracle.cluster(X, 0.08)
    Xf, lab = r["X"].astype(np.float32), r["labels"]
    assert theorem47.violations(Xf, lab, 0.08) == 0 == _brute(Xf, lab, 0.08)
    merged = np.where(lab == 1, 0, lab)
    assert theorem47.violations(Xf, merged, 0.08) == _brute(Xf, merged, 0.08) > 0
    split = lab.copy()
    big = np.bincount(lab).argmax()
    idx = np.nonzero(lab == big)[0]
    split[idx[: len(idx) // 2]] = lab.max() + 1
    assert theorem47.violations(Xf, split, 0.08) == _brute(Xf, split, 0.08) > 0


def test_checker_catches_close_clusters():
    X = np.array([[0.1, 0.1], [0.1, 0.1], [0.14, 0.1], [0.9, 0.9]], np.float32)
    assert theorem47.violations(X, np.array([0, 0, 1, 2]), 0.05) == 2   # 0.04 apart, different labels
    assert theorem47.violations(X, np.array([0, 0, 0, 1]), 0.05) == 0
    assert theorem47.violations(X, np.array([0, 0, 0, 0]), 0.05) == 3   # 0.9 point with all three
