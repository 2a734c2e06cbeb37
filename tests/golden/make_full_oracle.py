"""Write full-clustering goldens from the fp64 oracle (no GPU, no product code).

    python tests/golden/make_full_oracle.py C4-d2 C4-d5 C4-d10 C4-d15 C4-d20 C3

For each named BASELINE.json workload (seed 0, datagen recipe, DESIGN.md "Input
recipe") this runs ``oracle.cluster`` -- the plain O(T n^2 d) definition of
SynC iterated with Eq.1 and stopped by Def 4.2 in its grid form
(L108, L252) -- and stores under tests/golden/full/<cfg>_s<seed>.npz:

  iters         number of Eq.1 updates applied (Alg 4 semantics, reading R6)
  rc            oracle status (0 = converged, -6 = partition check failed)
  labels        canonical eps-graph component labels of the final state
                (Theorem 4.7; numbering by first occurrence, R14)
  n_clusters    max(labels)+1
  labels_sha256 sha256 of labels.astype('<i4').tobytes()
  sample_idx    4096 sampled point indices (rng seeded 12345), sorted
  sample_X      their final fp64 coordinates
  oracle_sha    sha256 of oracle/oracle.c at generation time
  seconds       oracle wall time, threads = OMP_NUM_THREADS / nproc

Only ``oracle`` and ``datagen`` (which holds no arithmetic of the method) are
imported; nothing here comes from the CUDA path (task rule (3)).
"""
from __future__ import annotations

import hashlib
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from paper_conf_edbt_jorgensena23_b200 import datagen  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "full")


def oracle_sha() -> str:
    with open(os.path.join(ROOT, "oracle", "oracle.c"), "rb") as f:
        return hashlib.sha256(f.read()).hexdigest()


def make(name: str, seed: int = 0) -> str:
    cfg = datagen.make_config(name)
    X = cfg.generate(seed)
    t0 = time.time()
    r = oracle.cluster(X, cfg.eps)
    dt = time.time() - t0
    labels = r["labels"].astype(np.int32)
    rng = np.random.default_rng(12345)
    m = min(4096, cfg.n)
    idx = np.sort(rng.choice(cfg.n, size=m, replace=False)).astype(np.int64)
    os.makedirs(OUT, exist_ok=True)
    path = os.path.join(OUT, f"{name}_s{seed}.npz")
    np.savez_compressed(
        path, config=name, seed=seed, n=cfg.n, d=cfg.d, eps=np.float32(cfg.eps),
        iters=r["iters"], rc=r["rc"], labels=labels, n_clusters=int(labels.max()) + 1,
        labels_sha256=hashlib.sha256(labels.astype("<i4").tobytes()).hexdigest(),
        sample_idx=idx, sample_X=r["X"][idx], oracle_sha=oracle_sha(), seconds=dt,
        threads=int(os.environ.get("OMP_NUM_THREADS", os.cpu_count() or 1)))
    print(f"{name} seed={seed}: rc={r['rc']} iters={r['iters']} clusters={labels.max() + 1} "
          f"{dt:.1f} s -> {path}", flush=True)
    return path


if __name__ == "__main__":
    for a in sys.argv[1:] or ["C1"]:
        make(a)
