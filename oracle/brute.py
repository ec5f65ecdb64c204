"""Brute-force checker for the oracle (TEST INFRASTRUCTURE ONLY).

Independent of gbdt_oracle.c: no sorted lists, no scans, no running accumulators.  For every
node of a tree produced by the oracle it enumerates EVERY admissible split of the node's
instances -- each attribute, each distinct present value v (high = present & x >= v, R11), each
missing direction -- sums g/h over the two sides as exact rationals
(fractions.Fraction of the fp64 inputs), evaluates Eq. 2 exactly (+lambda per R1) and
checks that the oracle's choice is the exact maximiser (ties by the R12 total order), that the
split/leaf decision obeys "gain > max(gamma, 0)", that node sums/counts are the
member sums and that leaf weights are -G/(H+lambda) (R3).  Intended for n < 20.
"""
from __future__ import annotations

from fractions import Fraction
import math

import numpy as np


def _grad(loss, yhat, y):
    if loss == "squared":
        return 2.0 * (yhat - y), np.full_like(yhat, 2.0)
    p = 1.0 / (1.0 + np.exp(-yhat))
    return p - y, np.maximum(p * (1.0 - p), 1e-16)  # Eq. 1, reading R5


def _gain_exact(GL, HL, G, H, lam):
    GR, HR = G - GL, H - HL
    return Fraction(1, 2) * (GL * GL / (HL + lam) + GR * GR / (HR + lam) - G * G / (H + lam))


def check_tree(X, y, yhat, tree, params):
    """X dense float with NaN; tree = oracle nodes of ONE tree (structured array, heap order).
    Returns (list_of_failures, yhat_after)."""
    loss, d = params["loss"], int(params["max_depth"])
    lam = Fraction(float(params["lam"]))
    thr = Fraction(max(float(params["gamma"]), 0.0))
    g, h = _grad(loss, np.asarray(yhat, np.float64), np.asarray(y, np.float64))
    gF = [Fraction(float(v)) for v in g]
    hF = [Fraction(float(v)) for v in h]
    n, m = X.shape
    fails = []
    members = {0: list(range(n))}
    leaf_of = np.zeros(n, np.int64)
    for k in range(tree.shape[0]):
        if k not in members:
            if tree[k]["heap_id"] == k:
                fails.append(f"node {k} present in oracle tree but not reachable")
            continue
        mem = members[k]
        node = tree[k]
        if node["heap_id"] != k:
            fails.append(f"node {k} missing from oracle tree")
            continue
        G = sum((gF[i] for i in mem), Fraction(0))
        H = sum((hF[i] for i in mem), Fraction(0))
        if node["count"] != len(mem):
            fails.append(f"node {k}: count {node['count']} != {len(mem)}")
        if not math.isclose(float(node["G"]), float(G), rel_tol=1e-12, abs_tol=1e-12):
            fails.append(f"node {k}: G {node['G']} != {float(G)}")
        if not math.isclose(float(node["H"]), float(H), rel_tol=1e-12, abs_tol=1e-12):
            fails.append(f"node {k}: H {node['H']} != {float(H)}")
        depth = int(math.floor(math.log2(k + 1)))
        # enumerate every admissible split
        cands = []
        if depth < d:
            for a in range(m):
                xs = X[mem, a]
                present = ~np.isnan(xs)
                n_miss = int((~present).sum())
                for v in sorted(set(np.float32(xs[present]).tolist()), reverse=True):
                    for dr in ((0, 1) if n_miss > 0 else (0,)):
                        hi = [i for i, x in zip(mem, xs) if (not np.isnan(x) and np.float32(x) >= v)
                              or (np.isnan(x) and dr == 1)]
                        if len(hi) < 1 or len(mem) - len(hi) < 1:
                            continue
                        GL = sum((gF[i] for i in hi), Fraction(0))
                        HL = sum((hF[i] for i in hi), Fraction(0))
                        cands.append((_gain_exact(GL, HL, G, H, lam), a, float(v), dr, frozenset(hi)))
        best = None
        if cands:
            gmax = max(c[0] for c in cands)
            ties = [c for c in cands if c[0] == gmax]
            ties.sort(key=lambda c: (c[1], -c[2], c[3]))  # R12: attr asc, value desc, dir low first
            best = ties[0]
        should_split = best is not None and best[0] > thr
        if node["is_leaf"]:
            if should_split and not _near(best[0], thr):
                fails.append(f"node {k}: oracle leaf but brute best gain {float(best[0])} > thr")
            w = -float(G) / (float(H) + float(lam))
            if not math.isclose(float(node["weight"]), w, rel_tol=1e-12, abs_tol=1e-15):
                fails.append(f"node {k}: weight {node['weight']} != {w}")
            for i in mem:
                leaf_of[i] = k
            continue
        if not should_split and not (best is not None and _near(best[0], thr)):
            fails.append(f"node {k}: oracle split but brute says leaf")
            continue
        choice = (int(node["attr"]), float(node["split_value"]), int(node["default_left"]))
        match = [c for c in cands if (c[1], c[2], c[3]) == choice]
        if not match:
            fails.append(f"node {k}: oracle choice {choice} is not an admissible split")
            continue
        cg = match[0][0]
        if cg != best[0]:
            rel = abs(float(cg - best[0])) / max(abs(float(best[0])), 1e-300)
            if rel > 1e-9:
                fails.append(f"node {k}: oracle choice {choice} gain {float(cg)} < brute best "
                             f"{(best[1], best[2], best[3])} {float(best[0])}")
        # an exact rational tie may be split by fp64 rounding of the two sides' sums, so any
        # member of the exact-tie set is accepted here; the R12 tie rule itself is pinned on
        # fp-exact ties (duplicate columns, Appendix A tie variant) in test_oracle_pins.py
        if not math.isclose(float(node["gain"]), float(cg), rel_tol=1e-9, abs_tol=1e-15):
            fails.append(f"node {k}: gain {node['gain']} != exact {float(cg)}")
        hi = match[0][4]
        members[2 * k + 1] = [i for i in mem if i in hi]
        members[2 * k + 2] = [i for i in mem if i not in hi]
    w = np.array([float(tree[k]["weight"]) for k in leaf_of])
    return fails, np.asarray(yhat, np.float64) + float(params["eta"]) * w


def _near(gain, thr):
    return abs(float(gain - thr)) <= 1e-9 * max(abs(float(gain)), 1e-300)
