"""Full-clustering parity at BASELINE sizes against cached full-oracle goldens.

The goldens (tests/golden/full/<cfg>_s0.npz) are written by tests/golden/make_full_oracle.py,
which runs only oracle.cluster (the O(T n^2 d) definition: Eq.1 L68 + Def 4.2 L108 in its grid
form L252) on the CPU; no value in them comes from the CUDA path.  Bars (north_star):
  * canonical labels identical to the oracle's (elementwise), equal iteration count;
  * final coordinates within 1e-4 of the oracle's fp64 ones on 4096 sampled points;
  * the complete Theorem 4.7 property (L133) over all n points (tests/theorem47.py).
"""
import glob
import hashlib
import os

import numpy as np
import pytest

from paper_conf_edbt_jorgensena23_b200 import datagen
from paper_conf_edbt_jorgensena23_b200 import eggsync as E
from tests import theorem47

pytestmark = pytest.mark.gpu
GOLD = os.path.join(os.path.dirname(__file__), "golden", "full")
REQUIRED = ["C1", "C3", "C4-d2", "C4-d5", "C4-d10", "C4-d15", "C4-d20"]


# C3's full oracle run costs ~5 h on 8 cores (O(T n^2 d), n = 1M): its golden is committed when
# that run has finished; until then the C3 case is skipped (never passed silently).
SLOW = {"C3"}


def _golden(name):
    p = os.path.join(GOLD, f"{name}_s0.npz")
    if not os.path.exists(p):
        if name in SLOW:
            pytest.skip(f"golden {p} not generated yet: tests/golden/make_full_oracle.py {name}")
        pytest.fail(f"missing golden {p}: run tests/golden/make_full_oracle.py {name}")
    return np.load(p)


@pytest.mark.parametrize("name", REQUIRED)
def test_full_clustering_matches_oracle(name):
    g = _golden(name)
    c = datagen.make_config(name)
    X = c.generate(int(g["seed"]))
    assert X.shape == (int(g["n"]), int(g["d"]))
    r = E.cluster(X, c.eps, coords=True)
    assert int(g["rc"]) == 0 and r["converged"]
    lab = r["labels"]
    assert hashlib.sha256(lab.astype("<i4").tobytes()).hexdigest() == str(g["labels_sha256"]) or \
        np.array_equal(lab, g["labels"]), \
        f"labels differ at {np.nonzero(lab != g['labels'])[0][:10]} ({int((lab != g['labels']).sum())} points)"
    assert np.array_equal(lab, g["labels"])
    assert r["iters"] == int(g["iters"]), (r["iters"], int(g["iters"]))
    idx = g["sample_idx"]
    err = float(np.abs(r["coords"][idx].astype(np.float64) - g["sample_X"]).max())
    assert err <= 1e-4, err
    assert theorem47.violations(r["coords"], lab, c.eps) == 0


def test_goldens_are_oracle_outputs():
    """Every stored golden names the oracle source it came from (sha256 of oracle/oracle.c) and
    was produced by a converged oracle run."""
    for p in sorted(glob.glob(os.path.join(GOLD, "*.npz"))):
        g = np.load(p)
        assert len(str(g["oracle_sha"])) == 64 and int(g["rc"]) == 0, p
