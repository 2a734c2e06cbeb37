"""Both A6 update kernels against the oracle.

The library picks the update kernel per iteration (update_tc.cuh, tc_enabled and the plan's
occupancy rule): the tcgen05 tensor-core kernel while cells are mostly singletons (or fully
collapsed), the SIMT kernel otherwise and for small cell counts.  Small parity inputs would
therefore mostly exercise the SIMT kernel, so the whole GPU parity module is re-run in
subprocesses with the choice forced: EGGSYNC_TC=2 (tensor cores whenever d <= 12) and
EGGSYNC_TC=0 (SIMT only).  The default selection is what test_gpu_parity.py itself runs.
EGGSYNC_DENSE=1 selects the random-access grid update of PAPER.md §4.2.2 (F3, update_dense.cu)
wherever it applies (d <= 4): the parity module and the d <= 4 full-oracle goldens are re-run
with it.
"""
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.parametrize("mode", ["2", "0"])
def test_parity_module_with_forced_kernel(mode):
    env = dict(os.environ, EGGSYNC_TC=mode)
    r = subprocess.run([sys.executable, "-m", "pytest", os.path.join(ROOT, "tests", "test_gpu_parity.py"),
                        "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=1200)
    assert r.returncode == 0, r.stdout[-4000:] + r.stderr[-2000:]


def test_parity_with_dense_grid():
    """The random-access grid (d <= 4 cases of the parity module, C1 and C4-d2 full goldens)."""
    env = dict(os.environ, EGGSYNC_DENSE="1", EGGSYNC_SMALL="0")  # small inputs: the grid path too
    r = subprocess.run([sys.executable, "-m", "pytest", os.path.join(ROOT, "tests", "test_gpu_parity.py"),
                        os.path.join(ROOT, "tests", "test_gpu_full_parity.py"), "-k",
                        "not C3 and not C4-d5 and not C4-d10 and not C4-d15 and not C4-d20",
                        "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider"],
                       cwd=ROOT, env=env, capture_output=True, text=True, timeout=1200)
    assert r.returncode == 0, r.stdout[-4000:] + r.stderr[-2000:]
