"""Pins for the CPU oracle against what the paper and the mathematics fix (no GPU).

Each test names the passage it follows.  None of the expected values below comes from the
CUDA path: they are the paper's printed numbers (tests/golden/*.json, cited), hand-derived
fractions (Appendix A), closed forms, an independent exhaustive search (oracle/brute.py), or
scikit-learn's CART (a library routine the method reduces to for squared loss, lambda=0).
"""
import json
import math
import os

import numpy as np
import pytest

from datagen import synth
from oracle import brute, oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


# ------------------------------------------------------------------ layout
def test_table1_sorted_lists():
    gd = _gold("table1_sorted.json")
    p = synth.table1()
    col_ptr, val, ins = oracle.presort(p.indptr, p.indices, p.values, p.n, p.m)
    for a in range(p.m):
        got = list(zip(ins[col_ptr[a]:col_ptr[a + 1]].tolist(), val[col_ptr[a]:col_ptr[a + 1]].tolist()))
        exp = [(i, v) for i, v in gd["sorted"][str(a)]]
        assert [round(v, 6) for _, v in got] == [round(v, 6) for _, v in exp]      # descending values
        # ties compared as multisets within equal-value runs (R9); ours are ascending ids
        for v in set(round(v, 6) for _, v in exp):
            assert sorted(i for i, x in got if round(x, 6) == v) == sorted(i for i, x in exp if round(x, 6) == v)
            run = [i for i, x in got if round(x, 6) == v]
            assert run == sorted(run)


def test_presort_matches_lexsort_random():
    rng = np.random.default_rng(7)
    X = rng.integers(0, 6, size=(200, 5)).astype(np.float64) - 2.0
    X[rng.uniform(size=X.shape) < 0.3] = np.nan
    X[0, 0] = -0.0
    p = synth.from_dense("r", X, np.zeros(200), {})
    col_ptr, val, ins = oracle.presort(p.indptr, p.indices, p.values, p.n, p.m)
    for a in range(p.m):
        rows = np.where(~np.isnan(X[:, a]))[0]
        v = X[rows, a] + 0.0  # -0.0 -> +0.0
        order = np.lexsort((rows, -v))
        assert np.array_equal(ins[col_ptr[a]:col_ptr[a + 1]], rows[order])
        assert np.array_equal(val[col_ptr[a]:col_ptr[a + 1]], v[order].astype(np.float32))
    assert not np.signbit(val[val == 0]).any()


def test_rle_example_p233():
    gd = _gold("rle_p233.json")
    rv, rl = oracle.rle_encode(np.array(gd["values"], np.float32))
    assert [(round(float(v), 6), int(l)) for v, l in zip(rv, rl)] == [tuple(r) for r in gd["runs"]]


def test_fig1_segmented_prefix_sum():
    gd = _gold("fig1_scan.json")
    out = oracle.seg_scan(np.array(gd["gradient"]), np.array(gd["head"]))
    np.testing.assert_allclose(out, gd["prefix"], rtol=0, atol=gd["tol"])


# ------------------------------------------------------------------ Eq. 1 closed forms
def test_gradients_closed_forms_at_zero():
    y = np.array([0, 1, 0, 1, 0.25], np.float32)
    g, h = oracle.gradients("squared", np.zeros(5), y)
    np.testing.assert_array_equal(g, -2.0 * y.astype(np.float64))
    np.testing.assert_array_equal(h, 2.0)
    g, h = oracle.gradients("logistic", np.zeros(5), y)
    np.testing.assert_allclose(g, 0.5 - y.astype(np.float64), rtol=0, atol=1e-16)
    np.testing.assert_allclose(h, 0.25, rtol=0, atol=1e-16)


@pytest.mark.parametrize("loss", ["squared", "logistic"])
def test_gradients_are_loss_derivatives(loss):
    rng = np.random.default_rng(3)
    yh = rng.normal(0, 2, 64)
    y = (rng.uniform(size=64) < 0.5).astype(np.float32)
    if loss == "squared":
        lf = lambda z: (y - z) ** 2
    else:
        lf = lambda z: -(y * np.log(1 / (1 + np.exp(-z))) + (1 - y) * np.log(1 - 1 / (1 + np.exp(-z))))
    eps = 1e-4
    gfd = (lf(yh + eps) - lf(yh - eps)) / (2 * eps)
    hfd = (lf(yh + eps) - 2 * lf(yh) + lf(yh - eps)) / eps ** 2
    g, h = oracle.gradients(loss, yh, y)
    np.testing.assert_allclose(g, gfd, rtol=1e-6, atol=1e-8)
    np.testing.assert_allclose(h, hfd, rtol=1e-4, atol=1e-6)


# ------------------------------------------------------------------ Appendix A (Table I, Eq. 2)
def _tree(nodes, t):
    return {int(k): nodes[t, k] for k in range(nodes.shape[1]) if nodes[t, k]["heap_id"] == k}


def test_appendix_a_hand_example():
    gd = _gold("appendixA.json")
    p = synth.table1(loss="squared", d=2, T=2, lam=1.0, gamma=0.0, eta=1.0)
    nodes, margin, _ = oracle.train(p)
    tol = gd["tol_rel"]
    for t, key in ((0, "tree0"), (1, "tree1")):
        tr = _tree(nodes, t)
        e = gd[key]
        r = tr[0]
        assert not r["is_leaf"]
        assert (r["attr"], round(float(r["split_value"]), 6), r["default_left"]) == \
            (e["root_attr"], e["root_value"], e["root_default_left"])
        assert math.isclose(r["gain"], e["root_gain"], rel_tol=tol)
        assert tr[1]["is_leaf"] and tr[2]["is_leaf"] and set(tr) == {0, 1, 2}
        assert tr[1]["weight"] == 0.0 and math.isclose(tr[2]["weight"], e["low_weight"], rel_tol=tol)
    np.testing.assert_allclose(margin, gd["margin_after_tree1"], rtol=tol, atol=1e-15)
    n1, m1, _ = oracle.train(p, params=dict(n_trees=1))
    np.testing.assert_allclose(m1, gd["margin_after_tree0"], rtol=tol, atol=1e-15)


def test_appendix_a_exact_tie_lowest_attribute_wins():
    gd = _gold("appendixA.json")["tie_variant"]
    p = synth.table1(loss="squared", d=1, T=1, lam=1.0, eta=1.0)
    keep = p.indices != 0                                 # remove a1 entirely (all missing)
    counts = np.add.reduceat(keep.astype(np.int64), p.indptr[:-1]) if p.nnz else np.zeros(p.n)
    indptr = np.concatenate([[0], np.cumsum(counts)]).astype(np.int64)
    q = synth.Problem("t1noa1", p.n, p.m, indptr, p.indices[keep], p.values[keep], p.labels, p.params)
    nodes, _, _ = oracle.train(q)
    r = nodes[0, 0]
    assert (r["attr"], round(float(r["split_value"]), 6), r["default_left"]) == \
        (gd["root_attr"], gd["root_value"], gd["root_default_left"])
    assert math.isclose(r["gain"], gd["root_gain"], rel_tol=1e-12)


def test_gamma_is_strict_threshold():
    # the Appendix A root gain is 32/45; gamma exactly at it must NOT split (P:165 strict >)
    p = synth.table1(loss="squared", d=2, T=1, lam=1.0, eta=1.0)
    nodes, _, _ = oracle.train(p, params=dict(gamma=oracle.gain(0.0, 4.0, -4.0, 8.0, 1.0)))
    assert nodes[0, 0]["is_leaf"] == 1
    nodes, _, _ = oracle.train(p, params=dict(gamma=0.71))
    assert nodes[0, 0]["is_leaf"] == 0


# ------------------------------------------------------------------ exhaustive search, n < 20
@pytest.mark.parametrize("seed", range(12))
@pytest.mark.parametrize("loss", ["squared", "logistic"])
def test_bruteforce_small(seed, loss):
    gamma = 0.05 if seed % 4 == 3 else 0.0
    lam = 0.0 if (seed % 5 == 4 and loss == "squared") else 1.0
    p = synth.random_small(seed, n=8 + seed % 11, m=3 + seed % 3, nan_frac=0.25, n_distinct=3 + seed % 4,
                           loss=loss, d=3, T=2, lam=lam, gamma=gamma, eta=0.5)
    nodes, margin, _ = oracle.train(p)
    X = p.dense()
    yhat = np.zeros(p.n)
    for t in range(nodes.shape[0]):
        fails, yhat = brute.check_tree(X, p.labels, yhat, nodes[t], p.params)
        assert not fails, fails
    np.testing.assert_array_equal(margin, yhat)


# ------------------------------------------------------------------ library special case: CART
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_squared_lambda0_is_cart(seed):
    from sklearn.tree import DecisionTreeRegressor
    rng = np.random.default_rng(seed)
    n, m, d = 300, 5, 4
    X = rng.uniform(-1, 1, size=(n, m)).astype(np.float32).astype(np.float64)
    y = np.sin(3 * X[:, 0]) + X[:, 1] * X[:, 2] + 0.1 * rng.normal(size=n)
    p = synth.from_dense("cart", X, y, dict(loss="squared", max_depth=d, n_trees=2, lam=0.0, gamma=0.0,
                                            eta=1.0, base_margin=0.0))
    nodes, margin, _ = oracle.train(p)
    y32 = p.labels.astype(np.float64)
    resid = y32.copy()
    pred = np.zeros(n)
    for t in range(2):
        sk = DecisionTreeRegressor(max_depth=d, random_state=0).fit(X.astype(np.float32), resid)
        one = oracle.predict(nodes[t:t + 1], p.indptr, p.indices, p.values, eta=1.0)
        # same partition of the instances into leaves ...
        leaves_sk = sk.apply(X.astype(np.float32))
        groups_sk = {frozenset(np.where(leaves_sk == l)[0]) for l in np.unique(leaves_sk)}
        groups_or = {frozenset(np.where(one == v)[0]) for v in np.unique(one)}
        assert groups_sk == groups_or
        # ... and leaf value = mean residual
        np.testing.assert_allclose(one, sk.predict(X.astype(np.float32)), rtol=0, atol=1e-12)
        pred = pred + one
        resid = y32 - pred
    np.testing.assert_allclose(margin, pred, rtol=0, atol=1e-12)


# ------------------------------------------------------------------ invariants on C1
def test_c1_invariants_and_duplicate_column():
    p = synth.c1()
    nodes, margin, _ = oracle.train(p)
    d = p.params["max_depth"]
    lam = p.params["lam"]
    for t in range(nodes.shape[0]):
        tr = _tree(nodes, t)
        assert tr[0]["count"] == p.n
        leaves = 0
        for k, nd in tr.items():
            assert int(math.floor(math.log2(k + 1))) <= d
            if nd["is_leaf"]:
                leaves += nd["count"]
                assert nd["weight"] == -nd["G"] / (nd["H"] + lam)
            else:
                hi, lo = tr[2 * k + 1], tr[2 * k + 2]
                assert hi["count"] + lo["count"] == nd["count"] and hi["count"] >= 1 and lo["count"] >= 1
                assert math.isclose(hi["G"] + lo["G"], nd["G"], rel_tol=1e-12, abs_tol=1e-9)
                assert math.isclose(hi["H"] + lo["H"], nd["H"], rel_tol=1e-12)
                assert nd["gain"] > max(p.params["gamma"], 0.0)
                assert nd["attr"] != 7              # a7 is an exact copy of a0: ties go to a0 (R12)
        assert leaves == p.n
    pred = oracle.predict(nodes, p.indptr, p.indices, p.values, eta=p.params["eta"])
    np.testing.assert_array_equal(pred, margin)    # prediction by traversal == SmartGD margin


def test_follow_mode_self_consistent():
    p = synth.c1(n=400)
    nodes, margin, st = oracle.train(p)
    n2, m2, st2 = oracle.train(p, follow=nodes)
    assert st2["mismatch"] == 0 and st2["near_tie"] == 0 and st2["exact"] > 0
    np.testing.assert_array_equal(m2, margin)
    for f in ("attr", "split_value", "default_left", "is_leaf", "count", "weight"):
        np.testing.assert_array_equal(n2[f], nodes[f])


def test_follow_mode_flags_a_wrong_split():
    p = synth.c1(n=400)
    nodes, _, _ = oracle.train(p)
    bad = nodes.copy()
    bad[0, 0]["attr"] = 3 if nodes[0, 0]["attr"] != 3 else 4
    bad[0, 0]["split_value"] = np.float32(0.5)
    _, _, st = oracle.train(p, follow=bad)
    assert st["mismatch"] >= 1


# ------------------------------------------------------------------ follow-mode acceptance bands
# The north_star exempts only near-ties: a different (attr, value, dir) is accepted iff its gain is
# within 1e-6 relative of the oracle's best; a different split/leaf decision iff the best gain is
# within max(1e-6 |gain|, 1e-12 S) of gamma (SURVEY §8(c) "Follow mode").  These pins construct
# gaps just inside and just outside each band, priced by exact rational Eq. 2 (brute force), so a
# band set 10x too wide or too narrow fails one of them.
from fractions import Fraction


def _exact_gain(g, h, hi, lam):
    G, H = sum(g), sum(h)
    GL = sum(g[i] for i in hi)
    HL = sum(h[i] for i in hi)
    GR, HR = G - GL, H - HL
    return Fraction(1, 2) * (GL * GL / (HL + lam) + GR * GR / (HR + lam) - G * G / (H + lam))


def _two_split_problem(delta, K=1000):
    """Squared loss, lambda=1, depth 1, yhat=0.  a0 sends {0..K-1} high; a1 sends {0..K-1, 2K}
    high.  Instances 0..K-1 have y=1, K..2K-1 y=0, instance 2K has y=delta: delta moves the gain
    of a1 relative to a0 continuously (delta=0 favours a0, delta=1 favours a1)."""
    n = 2 * K + 1
    y = np.zeros(n, np.float32)
    y[:K] = 1.0
    y[2 * K] = np.float32(delta)
    X = np.zeros((n, 2))
    X[:K, 0] = 1.0
    X[:K, 1] = 1.0
    X[2 * K, 1] = 1.0
    p = synth.from_dense("ties", X, y, dict(loss="squared", max_depth=1, n_trees=1, lam=1.0,
                                             gamma=0.0, eta=1.0, base_margin=0.0))
    g = [Fraction(-2.0 * float(v)) for v in p.labels]    # P:193 at yhat = 0
    h = [Fraction(2)] * n
    lam = Fraction(1)
    ga0 = _exact_gain(g, h, range(K), lam)
    ga1 = _exact_gain(g, h, list(range(K)) + [2 * K], lam)
    return p, ga0, ga1


def _delta_for_gap(gap):
    """float32 delta with exact gain(a1) = gain(a0) * (1 - rel), rel as close to `gap` as fp32 allows."""
    lo, hi = 0.0, 1.0
    for _ in range(60):
        mid = float(np.float32((lo + hi) / 2))
        _, a0, a1 = _two_split_problem(mid)
        if 1 - a1 / a0 > gap:
            lo = mid
        else:
            hi = mid
        if lo == hi or mid in (lo, hi) and hi - lo < 1e-7:
            break
    return lo


def _follow_with(nodes, **root):
    f = nodes.copy()
    for k, v in root.items():
        f[0, 0][k] = v
    return f


@pytest.mark.parametrize("gap,status", [(1e-7, 1), (5e-7, 1), (2e-6, 2), (1e-5, 2)])
def test_follow_near_tie_band(gap, status):
    p, a0, a1 = _two_split_problem(_delta_for_gap(gap))
    rel = float(1 - a1 / a0)
    assert 0.5 * gap <= rel <= 2.0 * gap, rel            # the construction hit the intended gap
    nodes, _, st = oracle.train(p)
    assert (nodes[0, 0]["attr"], nodes[0, 0]["is_leaf"]) == (0, 0) and st["mismatch"] == 0
    follow = _follow_with(nodes, attr=1, split_value=np.float32(1.0), default_left=0)
    fn, _, st = oracle.train(p, follow=follow)
    assert fn[0, 0]["follow_status"] == status, (rel, fn[0, 0]["follow_status"])
    if status == 1:                                      # accepted: training continues with a1
        assert st["near_tie"] == 1 and fn[0, 0]["attr"] == 1 and fn[0, 1]["count"] == 1001


def _table1_root():
    p = synth.table1(loss="squared", d=1, T=1, lam=1.0, eta=1.0)
    nodes, _, _ = oracle.train(p)
    return p, nodes, Fraction(32, 45)                    # Appendix A root gain


@pytest.mark.parametrize("rel,status", [(1e-8, 1), (5e-7, 1), (3e-6, 2), (1e-4, 2)])
def test_follow_gamma_band_oracle_splits_follower_leaf(rel, status):
    """gamma just below the best gain: the oracle splits, the followed model made a leaf."""
    p, nodes, g = _table1_root()
    leaf = nodes.copy()
    leaf[0] = np.zeros_like(leaf[0])
    leaf[0]["heap_id"] = -1
    leaf[0, 0] = nodes[0, 0]
    leaf[0, 0]["is_leaf"] = 1
    fn, _, _ = oracle.train(p, params=dict(gamma=float(g) * (1 - rel)), follow=leaf)
    assert fn[0, 0]["follow_status"] == status


@pytest.mark.parametrize("rel,status", [(1e-8, 1), (5e-7, 1), (3e-6, 2), (1e-4, 2)])
def test_follow_gamma_band_oracle_leaf_follower_splits(rel, status):
    """gamma just above the best gain: the oracle makes a leaf, the followed model split."""
    p, nodes, g = _table1_root()
    own, _, _ = oracle.train(p, params=dict(gamma=float(g) * (1 + rel)))
    assert own[0, 0]["is_leaf"] == 1
    fn, _, _ = oracle.train(p, params=dict(gamma=float(g) * (1 + rel)), follow=nodes)
    assert fn[0, 0]["follow_status"] == status


def _flat_problem(eps):
    """gamma = 0 and one admissible split whose gain is a tiny remnant of cancellation: the high
    half has y = 1 + eps, the low half y = 1 (squared loss, lambda = 0, so the gain is the SSE
    reduction).  S = GL^2/HL + GR^2/HR ~ 4000 while the gain ~ 1000 eps^2."""
    K = 1000
    y = np.ones(2 * K, np.float32)
    y[:K] = np.float32(1.0 + eps)
    X = np.zeros((2 * K, 1))
    X[:K, 0] = 1.0
    return synth.from_dense("flat", X, y, dict(loss="squared", max_depth=1, n_trees=1, lam=0.0,
                                                gamma=0.0, eta=1.0, base_margin=0.0))


@pytest.mark.parametrize("eps,status", [(2.0 ** -23, 1), (1.5e-6, 1), (5e-6, 2), (2.0 ** -13, 2)])
def test_follow_gamma_band_cancellation_floor(eps, status):
    """The 1e-12 S floor of the gamma band: gains of ~2e-15 S (one fp32 ulp of label difference)
    and ~3e-13 S are within the band whichever way the followed model decided; gains of ~3e-12 S
    and ~7e-9 S are real splits and a followed leaf is a mismatch."""
    p = _flat_problem(eps)
    nodes, _, _ = oracle.train(p)
    g = [Fraction(-2.0 * float(v)) for v in p.labels]
    h = [Fraction(2)] * p.n
    gain = _exact_gain(g, h, range(1000), Fraction(0))
    GL, G = sum(g[:1000]), sum(g)
    S = GL * GL / 2000 + (G - GL) ** 2 / 2000
    ratio = float(gain / S)
    assert (ratio < 0.5e-12) if status == 1 else (2e-12 < ratio < 1e-6), ratio
    ref = synth.from_dense("ref", np.array([[1.0], [0.0]]), np.array([1.0, 0.0]), dict(p.params))
    split_tree, _, _ = oracle.train(ref)                 # a 1-split tree on a0 >= 1 (same heap shape)
    if nodes[0, 0]["is_leaf"]:                           # fp64 rounding decided "leaf": follow a split
        follow = split_tree.copy()
        follow[0, 0]["split_value"] = np.float32(1.0)
    else:                                                # it decided "split": follow a leaf
        follow = nodes.copy()
        follow[0, 1:] = np.zeros_like(follow[0, 1:])
        follow[0, 1:]["heap_id"] = -1
        follow[0, 0]["is_leaf"] = 1
    assert status == 1 or nodes[0, 0]["is_leaf"] == 0    # a 1e-9 S gain survives fp64 rounding
    fn, _, _ = oracle.train(p, follow=follow)
    assert fn[0, 0]["follow_status"] == status


@pytest.mark.parametrize("off,status", [(0.3e-12, 1), (3e-12, 2)])
def test_follow_gamma_band_cancellation_floor_follower_splits(off, status):
    """The same floor from the other side: gamma sits `off` S above a tiny gain (~3e-12 S, so
    1e-6 |gain| is far below 1e-12 S): the oracle makes a leaf, the followed model split."""
    p = _flat_problem(5e-6)
    nodes, _, _ = oracle.train(p)
    assert nodes[0, 0]["is_leaf"] == 0
    g = [Fraction(-2.0 * float(v)) for v in p.labels]
    GL, G = sum(g[:1000]), sum(g)
    S = float(GL * GL / 2000 + (G - GL) ** 2 / 2000)
    gamma = float(nodes[0, 0]["gain"]) + off * S
    own, _, _ = oracle.train(p, params=dict(gamma=gamma))
    assert own[0, 0]["is_leaf"] == 1
    fn, _, _ = oracle.train(p, params=dict(gamma=gamma), follow=nodes)
    assert fn[0, 0]["follow_status"] == status
