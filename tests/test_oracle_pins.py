"""Pins of the fp64 oracle against what the paper and mathematics fix.

Every test here is CPU-only (`-m "not gpu"`).  Each pins a piece of
oracle/oracle.c to something other than itself: a closed form, the App.D
recurrence, a geometric derivation, an invariant, an independent formula
(Eq.5 vs Eq.1), or a hand-derived worked example (tests/golden/).
A plausible mistake (dropped 1/|N|, sin(p-q) instead of sin(q-p), strict < in
N_eps, Gauss-Seidel instead of Jacobi, wrong delta, wrong cell width or clamp,
criterion on the wrong state) fails at least one of them.
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
from paper_conf_edbt_jorgensena23_b200 import datagen

GOLD = json.load(open(os.path.join(os.path.dirname(__file__), "golden", "worked_examples.json")))


# ---------------------------------------------------------------- closed forms
def test_two_point_closed_form_eq1():
    """Eq.1 L68 with |N|=2: x' = x + sin(y-x)/2 (pins 1/|N|, p in N(p), sign, Jacobi)."""
    x = np.array([0.5, 0.5], np.float32)
    y = np.array([0.52, 0.53], np.float32)
    Xn, nbr, _ = oracle.step(np.stack([x, y]), 0.05)
    xd, yd = x.astype(np.float64), y.astype(np.float64)
    for i in range(2):
        assert Xn[0, i] == pytest.approx(xd[i] + 0.5 * math.sin(yd[i] - xd[i]), abs=1e-15)
        assert Xn[1, i] == pytest.approx(yd[i] + 0.5 * math.sin(xd[i] - yd[i]), abs=1e-15)
    assert nbr.tolist() == [2, 2]
    # SURVEY P1 digits (closed form evaluated on the fp64 inputs 0.5/0.52/0.53)
    Xn64, _, _ = oracle.step(np.array([[0.5, 0.5], [0.52, 0.53]], np.float64), 0.05)
    assert Xn64[0] == pytest.approx([0.5099993333, 0.5149977501], abs=1e-9)


def test_isolated_point_never_moves():
    """Eq.1: N(p)={p} -> sum sin(0)=0 (L68)."""
    X = np.array([[0.1, 0.1], [0.9, 0.9]], np.float32)
    Xn, nbr, f = oracle.step(X, 0.05, compute_f2=True)
    assert np.array_equal(Xn, X.astype(np.float64))
    assert nbr.tolist() == [1, 1]
    assert f == (1, 1, 1)


def test_app_d_gap_recurrence():
    """App.D: for two points moving together the per-dim gap obeys d' = d - sin(d)."""
    X = np.array([[0.30, 0.60, 0.45], [0.33, 0.58, 0.47]], np.float32)
    g = (X[1].astype(np.float64) - X[0].astype(np.float64))
    cur = X.astype(np.float64)
    for _ in range(6):
        cur, nbr, _ = oracle.step(cur, 0.05)
        assert nbr.tolist() == [2, 2]
        g = g - np.sin(g)
        assert cur[1] - cur[0] == pytest.approx(g, abs=1e-15)
    # the midpoint is preserved by symmetry (sin odd)
    assert (cur[0] + cur[1]) / 2 == pytest.approx((X[0].astype(np.float64) + X[1]) / 2, abs=1e-15)


def test_neighbourhood_is_inclusive():
    """L66: N_eps(p) = {q : ||p-q|| <= eps} -- a pair at exactly eps are neighbours."""
    e = np.float32(0.05)
    X = np.array([[0.0, 0.5], [e, 0.5]], np.float32)  # squared distance == eps^2 exactly in fp64
    _, nbr, _ = oracle.step(X, float(e))
    assert nbr.tolist() == [2, 2]
    X2 = np.array([[0.0, 0.5], [np.nextafter(e, np.float32(1)), 0.5]], np.float32)
    _, nbr2, _ = oracle.step(X2, float(e))
    assert nbr2.tolist() == [1, 1]


def test_eq5_identity_against_eq1():
    """Eq.5 L228-235 is a different formula for the same update:
    x + (cos x * sum sin q - sin x * sum cos q)/|N|  must equal the oracle's Eq.1 result."""
    rng = np.random.default_rng(3)
    X = (0.4 + 0.1 * rng.random((40, 4))).astype(np.float32)
    Xd = X.astype(np.float64)
    Xn, nbr, _ = oracle.step(X, 0.07)
    D2 = ((Xd[None, :, :] - Xd[:, None, :]) ** 2).sum(-1)
    M = D2 <= np.float64(np.float32(0.07)) ** 2
    assert M.sum(1).tolist() == nbr.tolist()
    S = M.astype(np.float64) @ np.sin(Xd)
    C = M.astype(np.float64) @ np.cos(Xd)
    eq5 = Xd + (np.cos(Xd) * S - np.sin(Xd) * C) / M.sum(1)[:, None]
    np.testing.assert_allclose(Xn, eq5, rtol=0, atol=1e-14)


def test_eq6_grid_split_reproduces_sum():
    """Eq.6: splitting the neighbourhood sum into full cells (summaries) and partial
    cells (point scan) gives the same sum.  Cells of width eps/(2 sqrt d) (L252)."""
    rng = np.random.default_rng(5)
    X = datagen.blobs(300, 2, 3, seed=5).astype(np.float64)
    eps = 0.1
    c = oracle.constants(eps, 2)
    cells = np.minimum(np.floor(X * c["inv_cw"]), c["w"] - 1).astype(np.int64)
    keys = cells[:, 0] * int(c["w"]) + cells[:, 1]
    e2 = c["eps2"]
    for p in rng.choice(300, 20, replace=False):
        total = np.zeros(2)
        for k in np.unique(keys):
            members = np.where(keys == k)[0]
            d2 = ((X[members] - X[p]) ** 2).sum(1)
            if (d2 <= e2).all():          # full cell -> its summary
                total += np.sin(X[members]).sum(0)
            elif (d2 <= e2).any():        # partial cell -> scan points
                total += np.sin(X[members[d2 <= e2]]).sum(0)
        d2all = ((X - X[p]) ** 2).sum(1)
        np.testing.assert_allclose(total, np.sin(X[d2all <= e2]).sum(0), rtol=1e-13)
    # and the oracle's neighbour counts agree with this brute force
    _, nbr, _ = oracle.step(X, eps)
    d2 = ((X[None] - X[:, None]) ** 2).sum(-1)
    assert nbr.tolist() == (d2 <= e2).sum(1).tolist()


# ------------------------------------------------------------------ constants
@pytest.mark.parametrize("eps", [0.025, 0.05, 0.1])
def test_delta_from_appendix_d_geometry(eps):
    """delta = delta1 + delta2 (App.D): delta1 solves eps^2 = (eps - delta1)^2 + (eps/4)^2
    (Eq.7, solved here by bisection, not by the closed form), delta2 = eps/2 - sin(eps/2)."""
    e = float(np.float32(eps))
    lo, hi = 0.0, e
    for _ in range(200):  # f(delta1) = (e - delta1)^2 + (e/4)^2 - e^2, decreasing on [0, e]
        mid = (lo + hi) / 2
        if (e - mid) ** 2 + (e / 4) ** 2 - e ** 2 > 0:
            lo = mid
        else:
            hi = mid
    d1 = (lo + hi) / 2
    d2 = e / 2 - math.sin(e / 2)
    c = oracle.constants(eps, 3)
    assert c["delta"] == pytest.approx(d1 + d2, rel=1e-12)
    assert c["ed2"] == pytest.approx((e + d1 + d2) ** 2, rel=1e-12)
    # the garbled App.D form (L392) is negative -- not the one used (R11)
    assert e - e * math.sqrt(15 / 16 + e / 2) - math.sin(e / 2) < 0


def test_delta_printed_values():
    """SURVEY P6 digits for delta(eps) (from L110)."""
    assert oracle.constants(0.05, 2)["delta"] == pytest.approx(0.0015903123, abs=1e-10)
    assert oracle.constants(0.1, 2)["delta"] == pytest.approx(0.0031962471, abs=1e-10)


@pytest.mark.parametrize("d", [1, 2, 3, 5, 10, 20])
def test_cell_diagonal_is_half_eps(d):
    """L252: c_w <= sqrt((eps/2)^2/d) so that the cell diagonal <= eps/2 (equality reading R1);
    Eq.4: w = ceil(1/c_w) cells per dimension."""
    c = oracle.constants(0.05, d)
    assert c["cw"] * math.sqrt(d) == pytest.approx(float(np.float32(0.05)) / 2, rel=1e-15)
    assert c["w"] == math.ceil(1.0 / c["cw"])


def test_cell_clamp_at_one():
    """R2: x = 1.0 belongs to the last cell w-1.  eps=0.5, d=4 -> c_w = 1/8 exactly, so
    1.0 * (1/c_w) = 8 = w and the clamp min(., w-1) decides (Eq.4 L151 garbled; DESIGN R2)."""
    c = oracle.constants(0.5, 4)
    assert c["cw"] == 0.125 and c["w"] == 8
    X = np.array([[1.0, 1.0, 1.0, 1.0], [0.9, 0.9, 0.9, 0.9]], np.float32)
    r = oracle.cluster(X, 0.5)
    # 0.9*8 = 7.2 -> cell 7 ; 1.0*8 = 8 -> clamped to 7 : same cell, so one cluster
    assert r["cell_labels"].tolist() == [0, 0]


# -------------------------------------------------------------- worked examples
@pytest.mark.parametrize("name", [k for k in GOLD if not k.startswith("_")])
def test_worked_examples(name):
    g = GOLD[name]
    X = np.array(g["points"], np.float32)
    r = oracle.cluster(X, g["eps"])
    assert r["rc"] == oracle.OK
    assert r["iters"] == g["iters"], g["cite"]
    assert r["labels"].tolist() == g["labels"], g["cite"]
    if "first_step_flags" in g:
        _, _, f = oracle.step(X, g["eps"], compute_f2=True)
        ff = g["first_step_flags"]
        assert f == (ff["F1_grid"], ff["F1_def42"], ff["F2"]), g["cite"]
    if "def42_iters" in g:
        r4 = oracle.cluster(X, g["eps"], term_mode=oracle.DEF42)
        assert r4["rc"] == oracle.OK and r4["iters"] == g["def42_iters"], g["cite"]
        assert r4["labels"].tolist() == g["labels"], g["cite"]


def test_bridge_chain_first_step_closed_form():
    """P4: a' = a + sin(b-a)/2 (|N(a)|=2), b' = b + (sin(a-b)+sin(c-b))/3 = b."""
    X = np.array([[0.40, 0.5], [0.44, 0.5], [0.48, 0.5]], np.float32)
    Xd = X.astype(np.float64)
    Xn, nbr, _ = oracle.step(X, 0.05)
    assert nbr.tolist() == [2, 3, 2]
    assert Xn[0, 0] == pytest.approx(Xd[0, 0] + math.sin(Xd[1, 0] - Xd[0, 0]) / 2, abs=1e-15)
    assert Xn[1, 0] == pytest.approx(Xd[1, 0] + (math.sin(Xd[0, 0] - Xd[1, 0]) + math.sin(Xd[2, 0] - Xd[1, 0])) / 3, abs=1e-15)


def test_second_term_mbr_geometry():
    """P5 by hand: ||p-q1|| in (eps, eps+delta] and dist(MBR{q1,q2},p) <= eps (L108-110)."""
    p, q1, q2 = (np.array(v, np.float32).astype(np.float64) for v in ([0.30, 0.495], [0.3512, 0.495], [0.349, 0.510]))
    c = oracle.constants(0.05, 2)
    d1 = math.dist(p, q1)
    assert c["eps"] < d1 <= c["eps"] + c["delta"]
    lo, hi = np.minimum(q1, q2), np.maximum(q1, q2)
    t = np.maximum(np.maximum(lo - p, 0), p - hi)
    assert math.sqrt((t ** 2).sum()) <= c["eps"]
    # the oracle's F2 fails on D^0, with term (i) satisfied in both forms
    _, _, f = oracle.step(np.stack([p, q1, q2]), 0.05, compute_f2=True)
    assert f == (1, 1, 0)


def test_second_term_needs_mbr_intersection():
    """Same shell distance as P5 but q's MBR far from p's ball: term (ii) holds (L104)."""
    X = np.array([[0.30, 0.495], [0.3512, 0.495], [0.3512, 0.480]], np.float32)
    _, _, f = oracle.step(X, 0.05, compute_f2=True)
    # dist(MBR, p) = 0.0512 > eps -> no violation; q1,q2 in the same cell? (19,27)/(19,28)
    assert f[2] == 1


# ------------------------------------------------------------------ invariants
def _rand_state(seed, n=60, d=3):
    return datagen.blobs(n, d, 3, seed=seed)


@pytest.mark.parametrize("seed", [0, 1])
def test_permutation_equivariance(seed):
    X = _rand_state(seed)
    perm = np.random.default_rng(seed).permutation(len(X))
    Xn, nbr, f = oracle.step(X, 0.1, compute_f2=True)
    Xp, nbrp, fp = oracle.step(X[perm], 0.1, compute_f2=True)
    np.testing.assert_allclose(Xp, Xn[perm], atol=1e-13)
    assert np.array_equal(nbrp, nbr[perm]) and f == fp


@pytest.mark.parametrize("seed", [0, 1])
def test_reflection_and_dimension_permutation(seed):
    """sin is odd: x -> 1-x maps the update to 1-x'; permuting dimensions permutes outputs."""
    X = _rand_state(seed).astype(np.float64)
    Xn, nbr, _ = oracle.step(X, 0.1)
    Xr, nbrr, _ = oracle.step(1.0 - X, 0.1)
    np.testing.assert_allclose(Xr, 1.0 - Xn, atol=1e-13)
    assert np.array_equal(nbr, nbrr)
    dp = [2, 0, 1]
    Xd, nbrd, _ = oracle.step(X[:, dp], 0.1)
    np.testing.assert_allclose(Xd, Xn[:, dp], atol=1e-13)
    assert np.array_equal(nbr, nbrd)


def test_translation_equivariance():
    X = (0.2 + 0.3 * datagen.uniform(50, 2, seed=4)).astype(np.float64)
    Xn, nbr, _ = oracle.step(X, 0.08)
    Xt, nbrt, _ = oracle.step(X + 0.25, 0.08)
    np.testing.assert_allclose(Xt - 0.25, Xn, atol=1e-12)
    assert np.array_equal(nbr, nbrt)


def test_update_stays_in_neighbourhood_range():
    """P7c: each x'_i lies in [min_{q in N(p)} q_i, max_{q in N(p)} q_i] (sin x <= x on [0,1])."""
    X = _rand_state(7, n=120, d=4).astype(np.float64)
    Xn, _, _ = oracle.step(X, 0.12)
    e2 = np.float64(np.float32(0.12)) ** 2
    d2 = ((X[None] - X[:, None]) ** 2).sum(-1)
    for p in range(len(X)):
        nb = X[d2[p] <= e2]
        assert (Xn[p] >= nb.min(0) - 1e-15).all() and (Xn[p] <= nb.max(0) + 1e-15).all()


def test_lemma_4_4_identical_neighbourhoods_contract():
    """Lemma 4.4: N(p) = N(q) implies per-dimension |p'-q'| <= |p-q| (App.B)."""
    rng = np.random.default_rng(11)
    X = np.concatenate([0.3 + 0.01 * rng.random((8, 3)), 0.7 + 0.01 * rng.random((6, 3))])
    Xn, nbr, _ = oracle.step(X, 0.05)
    for a in range(len(X)):
        for b in range(len(X)):
            if nbr[a] == nbr[b] and np.linalg.norm(X[a] - X[b]) <= 0.05:
                assert (np.abs(Xn[a] - Xn[b]) <= np.abs(X[a] - X[b]) + 1e-16).all()


def test_lemma_4_5_inequality():
    """Lemma 4.5 L120-127 (Eq.3) on a grid of (x, y) in (0,1], y > x."""
    v = np.linspace(0.01, 1.0, 80)
    for i, x in enumerate(v):
        for y in v[i + 1:]:
            assert math.sin(y - math.sin(y)) / math.sin(x - math.sin(x)) > math.sin(y) / math.sin(x)


# ------------------------------------------------------ termination & labels
@pytest.mark.parametrize("seed,d,eps", [(0, 2, 0.05), (1, 3, 0.08), (2, 5, 0.15)])
def test_theorem_4_7_at_termination(seed, d, eps):
    """Theorem 4.7: at the criterion, label(p)==label(q) <=> ||p-q|| <= eps on the final
    state, the eps-graph is a union of cliques, and K more updates change no neighbourhood
    (Def 4.1)."""
    X = datagen.blobs(200, d, 4, seed=seed)
    r = oracle.cluster(X, eps)
    assert r["rc"] == oracle.OK
    F = r["X"]
    e2 = np.float64(np.float32(eps)) ** 2
    A = ((F[None] - F[:, None]) ** 2).sum(-1) <= e2
    same = r["labels"][None, :] == r["labels"][:, None]
    assert np.array_equal(A, same)
    assert np.array_equal(r["labels"], r["cell_labels"])
    cur = F
    for _ in range(4):
        cur, _, _ = oracle.step(cur, eps)
        A2 = ((cur[None] - cur[:, None]) ** 2).sum(-1) <= e2
        assert np.array_equal(A2, A)


@pytest.mark.parametrize("seed,d", [(0, 2), (3, 3), (4, 5)])
def test_grid_and_def42_same_partition(seed, d):
    """Theorem 4.7: both first-term forms certify the final clustering, so partitions agree."""
    X = datagen.blobs(150, d, 3, seed=seed)
    a = oracle.cluster(X, 0.1, term_mode=oracle.GRID)
    b = oracle.cluster(X, 0.1, term_mode=oracle.DEF42)
    assert a["rc"] == b["rc"] == oracle.OK
    assert np.array_equal(a["labels"], b["labels"])
    assert b["iters"] <= a["iters"]


def test_grid_first_term_implies_def42_first_term():
    """L252: |cell(p)| = |N(p)| with diagonal <= eps/2 implies Def 4.2 term (i)."""
    for seed in range(6):
        X = datagen.blobs(120, 2, 3, seed=seed).astype(np.float64)
        cur = X
        for _ in range(8):
            nxt, _, f = oracle.step(cur, 0.1)
            if f[0] == 1:
                assert f[1] == 1
            cur = nxt


def test_eps_covering_everything():
    """P9: eps >= sqrt(d) -> one neighbourhood; all points converge to one cluster."""
    X = datagen.uniform(30, 2, seed=9)
    Xn, nbr, _ = oracle.step(X, 1.5)
    assert (nbr == 30).all()
    r = oracle.cluster(X, 1.5)
    assert r["rc"] == oracle.OK and (r["labels"] == 0).all()


def test_max_iters_not_converged():
    X = np.array([[0.40, 0.5], [0.44, 0.5], [0.48, 0.5]], np.float32)
    r = oracle.cluster(X, 0.05, max_iters=1)
    assert r["rc"] == oracle.NOT_CONVERGED and r["iters"] == 1


# ------------------------------------------------------- sampled variants
def test_step_sample_matches_full_step():
    X = datagen.blobs(400, 3, 4, seed=2)
    Xn, nbr, _ = oracle.step(X, 0.08)
    idx = np.array([0, 5, 17, 399, 200])
    Xs, ns = oracle.step_sample(X, 0.08, idx)
    np.testing.assert_array_equal(ns, nbr[idx])
    np.testing.assert_allclose(Xs, Xn[idx], atol=1e-15)


def test_terminal_violations_counts():
    X = np.array([[0.1, 0.1], [0.11, 0.1], [0.9, 0.9]], np.float32)
    assert oracle.terminal_violations(X, 0.05, [0, 0, 1], [0, 1, 2]) == 0
    assert oracle.terminal_violations(X, 0.05, [0, 1, 2], [0, 1, 2]) == 2
    assert oracle.terminal_violations(X, 0.05, [0, 0, 0], [2]) == 2


def test_generator_recipe():
    """datagen: shape, dtype, range, determinism, noise fraction."""
    a = datagen.blobs(5000, 4, 5, noise=0.1, seed=1)
    b = datagen.blobs(5000, 4, 5, noise=0.1, seed=1)
    assert a.dtype == np.float32 and a.shape == (5000, 4)
    assert a.min() == 0.0 and a.max() == 1.0
    assert np.array_equal(a, b)
    assert not np.array_equal(a, datagen.blobs(5000, 4, 5, noise=0.1, seed=2))


# ------------------------------------------------ Eq.2 cluster order parameter
def test_order_parameter_closed_forms():
    """Eq.2: isolated points give 1 (N={p}, e^0); a mutually-close pair gives (1+e^-a)/2;
    a chain 0, a, 2a (2a > eps) gives ((1+e^-a)/2 * 2 + (1+2e^-a)/3) / 3 (pins p in N(p),
    the 1/|N| inner mean, the 1/|D| outer mean, e^{-||.||} not e^{-||.||^2})."""
    X = np.array([[0.1, 0.1], [0.9, 0.9], [0.1, 0.9]], np.float32)
    r, rcp = oracle.order_parameter(X, 0.05)
    assert r == 1.0 and rcp.tolist() == [1.0, 1.0, 1.0]
    P = np.array([[0.5, 0.5], [0.52, 0.53]], np.float32)
    Pd = P.astype(np.float64)
    a = math.sqrt(((Pd[1] - Pd[0]) ** 2).sum())
    r, rcp = oracle.order_parameter(P, 0.05)
    assert r == pytest.approx((1 + math.exp(-a)) / 2, abs=1e-15)
    # pair + isolated point
    r, _ = oracle.order_parameter(np.vstack([P, [[0.9, 0.1]]]), 0.05)
    assert r == pytest.approx(((1 + math.exp(-a)) + 1) / 3, abs=1e-15)
    # chain: middle point sees both ends, the ends see only the middle
    C = np.array([[0.0], [0.03], [0.06]], np.float64)
    r, rcp = oracle.order_parameter(C, 0.05)
    e0, e1 = (1 + math.exp(-0.03)) / 2, (1 + 2 * math.exp(-0.03)) / 3
    assert rcp == pytest.approx([e0, e1, e0], abs=1e-15)
    assert r == pytest.approx((2 * e0 + e1) / 3, abs=1e-15)


def test_order_parameter_coincident_and_invariants():
    """Coincident neighbourhoods give r_c = 1 (L77 'r_c approach 1 when synchronized');
    0 < r_c <= 1; permutation invariance."""
    X = np.repeat(np.array([[0.2, 0.4, 0.6], [0.7, 0.1, 0.3]], np.float32), 5, axis=0)
    assert oracle.order_parameter(X, 0.05)[0] == 1.0
    Y = datagen.blobs(300, 3, 4, seed=5)
    r, rcp = oracle.order_parameter(Y, 0.08)
    assert 0.0 < r <= 1.0 and (rcp > 0).all() and (rcp <= 1).all()
    perm = np.random.default_rng(1).permutation(len(Y))
    r2, rcp2 = oracle.order_parameter(Y[perm], 0.08)
    assert r2 == pytest.approx(r, abs=1e-13)
    assert np.allclose(rcp2, rcp[perm], atol=1e-14, rtol=0)


def test_order_parameter_two_point_convergence():
    """App.D L392 + Eq.2: for a pair the gap g obeys g' = g - sin g, so r_c = (1+e^-|g|)/2
    rises towards 1 but never reaches it (L77, L95: 'r_c = 1 is never reached')."""
    X = np.array([[0.30, 0.60], [0.33, 0.58]], np.float64)
    g = X[1] - X[0]
    prev = 0.0
    for _ in range(3):  # gaps 3.6e-2, 7.8e-6, 8e-17: e^-|g| rounds to 1 after that
        r, _ = oracle.order_parameter(X, 0.05)
        assert r == pytest.approx((1 + math.exp(-math.sqrt((g ** 2).sum()))) / 2, abs=1e-14)
        assert prev < r and (r < 1.0 or math.sqrt((g ** 2).sum()) < 1e-15)
        prev = r
        X, _, _ = oracle.step(X, 0.05)
        g = g - np.sin(g)


def test_lambda_termination_stops_early_on_fig1_input():
    """Fig 1 (L89) / L95 / L298: Alg 1's r_c >= lambda (lambda = 0.999, L77) stops after 2
    updates on a bridge input whose state still fails Def 4.2 term (i) (the bridge points are
    eps-close to both clusters), while the exact criterion runs on until one cluster remains."""
    X = datagen.bridge()
    cur, t, r = X.copy(), 0, 0.0
    while r < 0.999:  # Alg 1 l.2-7 (r_c on D^t, update applied in the same iteration)
        r, _ = oracle.order_parameter(cur, 0.05)
        Xn, _, f = oracle.step(cur, 0.05)
        cur, t = Xn.astype(np.float32), t + 1
    assert t == 2 and 0.999 <= r < 0.9995
    _, _, f = oracle.step(cur, 0.05)
    assert f[0] == 0 and f[1] == 0  # not synchronized (Def 4.2 term i fails)
    res = oracle.cluster(X, 0.05)
    assert res["rc"] == oracle.OK and res["iters"] > 10
    assert len(set(res["labels"].tolist())) == 1


# ------------------------------------------- cell width below the L252 bound
def test_cw_factor_constants():
    """L252 only bounds c_w <= eps/(2 sqrt d); cw_factor f picks f*eps/(2 sqrt d), w = ceil(1/c_w) (Eq.4)."""
    c = oracle.constants(0.05, 2, 0.5)
    assert c["cw"] == pytest.approx(0.5 * 0.05 / (2 * math.sqrt(2)), rel=1e-7)
    assert c["w"] == math.ceil(1 / c["cw"]) == 114
    c1 = oracle.constants(0.05, 2)
    assert c1["w"] == 57 and c["delta"] == c1["delta"] and c["eps2"] == c1["eps2"]


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_cw_factor_same_clustering(seed):
    """Theorem 4.7 (L133-135) holds for any c_w <= eps/(2 sqrt d): the eps-components of the final
    state equal the verified state's cell partition (rc OK, no EPARTITION) and the partition is
    the same as at f = 1.  Halved cells nest in the f = 1 cells, so the grid criterion (L252) is
    stricter and never stops earlier."""
    X = datagen.blobs(600, 2, 5, seed=seed)
    r1 = oracle.cluster(X, 0.05)
    for f in (0.5, 0.3):
        rf = oracle.cluster(X, 0.05, cw_factor=f)
        assert rf["rc"] == oracle.OK
        assert np.array_equal(rf["labels"], r1["labels"])
        if f == 0.5:
            assert rf["iters"] >= r1["iters"]


def test_cw_factor_out_of_range():
    X = np.full((3, 2), 0.5, np.float32)
    for f in (0.0, 1.5, float("nan")):
        with pytest.raises(RuntimeError):
            oracle.cluster(X, 0.05, cw_factor=f)
