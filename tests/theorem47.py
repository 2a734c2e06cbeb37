"""Complete Theorem 4.7 check of a final clustering, for any n.

At the synchronization criterion every cluster's points pairwise lie within eps and points of
different clusters are more than eps apart: label(p) == label(q)  <=>  ||p - q|| <= eps.

Test infrastructure (numpy / scipy only; independent of both the CUDA path and the oracle):
  * intra-cluster: the MBR diagonal of each cluster <= eps implies every pair is within eps;
    a cluster whose diagonal exceeds eps is checked pair by pair (fp64);
  * inter-cluster: candidate cluster pairs are those whose MBR centres lie within
    eps + r_a + r_b (r = half MBR diagonal; a KD-tree query), then MINDIST(MBR_a, MBR_b) <= eps
    pairs are checked point by point in fp64 (the oracle's predicate, L66).
Returns the number of violating point pairs (0 = the theorem holds everywhere).
"""
from __future__ import annotations

import numpy as np


def _sq(a, b):
    t = a[:, None, :] - b[None, :, :]
    return (t * t).sum(-1)


def violations(X32, labels, eps: float) -> int:
    X = np.asarray(X32, np.float32).astype(np.float64)
    lab = np.asarray(labels, np.int64)
    n, d = X.shape
    e = float(np.float32(eps))
    e2 = e * e
    k = int(lab.max()) + 1
    order = np.argsort(lab, kind="stable")
    starts = np.searchsorted(lab[order], np.arange(k + 1))
    lo = np.full((k, d), np.inf)
    hi = np.full((k, d), -np.inf)
    np.minimum.at(lo, lab, X)
    np.maximum.at(hi, lab, X)
    bad = 0
    diag2 = ((hi - lo) ** 2).sum(1)
    for c in np.nonzero(diag2 > e2)[0]:           # intra-cluster pairs beyond eps
        P = X[order[starts[c]:starts[c + 1]]]
        bad += int((_sq(P, P) > e2).sum()) // 2
    from scipy.spatial import cKDTree
    cen = 0.5 * (lo + hi)
    rad = 0.5 * np.sqrt(diag2)
    live = np.nonzero(starts[1:] > starts[:-1])[0]   # labels that occur
    tree = cKDTree(cen[live])
    pairs = tree.query_pairs(e + 2.0 * rad[live].max() + 1e-12, output_type="ndarray")
    if len(pairs):
        a, b = live[pairs[:, 0]], live[pairs[:, 1]]
        gap = np.maximum(np.maximum(lo[a] - hi[b], lo[b] - hi[a]), 0.0)
        cand = (gap * gap).sum(1) <= e2               # MINDIST(MBR_a, MBR_b) <= eps
        for ca, cb in zip(a[cand], b[cand]):
            Pa = X[order[starts[ca]:starts[ca + 1]]]
            Pb = X[order[starts[cb]:starts[cb + 1]]]
            bad += int((_sq(Pa, Pb) <= e2).sum())
    return bad
