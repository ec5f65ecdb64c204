"""Parity helpers: compare a CUDA-path model with the CPU oracle (tests only).

Acceptance (BASELINE.json north_star): tree structure (split attribute, threshold, default
direction, leaf/internal) must match exactly except where the oracle's top two gains are within
1e-6 relative (follow mode accepts and counts those), and leaf weights / predictions must match
within 1e-5 relative (+1e-9 absolute floor, reading R23).
"""
import functools

import numpy as np

from datagen import synth
from oracle import oracle


@functools.lru_cache(maxsize=None)
def full_problem(name):
    """BASELINE.json config `name` at full size, generated once per test session."""
    return synth.make(name)

RTOL = 1e-5
ATOL = 1e-9


def compare(prob, nodes, margin, params=None, allow_near_ties=True):
    """Returns the oracle follow-mode stats; asserts parity."""
    return check(prob, nodes, margin, oracle.train(prob, params=params, follow=nodes), allow_near_ties)


def check(prob, nodes, margin, oracle_out, allow_near_ties=True):
    """Asserts parity of a CUDA model against an oracle follow-mode run (nodes, margin, stats)
    already computed on the same inputs with follow=nodes; returns the stats."""
    onodes, omargin, st = oracle_out
    assert st["mismatch"] == 0, f"{prob.name}: {st['mismatch']} node(s) differ from the oracle beyond near-ties: {st}"
    if not allow_near_ties:
        assert st["near_tie"] == 0, st
    present = nodes["heap_id"] >= 0
    assert np.array_equal(present, onodes["heap_id"] >= 0), "different node sets"
    for f in ("is_leaf", "attr", "default_left", "count"):
        assert np.array_equal(nodes[f][present], onodes[f][present]), f
    assert np.array_equal(nodes["split_value"][present], onodes["split_value"][present]), "split_value"
    leaf = present & (nodes["is_leaf"] == 1)
    np.testing.assert_allclose(nodes["weight"][leaf], onodes["weight"][leaf], rtol=RTOL, atol=ATOL)
    np.testing.assert_allclose(nodes["G"][present], onodes["G"][present], rtol=1e-6, atol=1e-7)
    np.testing.assert_allclose(nodes["H"][present], onodes["H"][present], rtol=1e-6, atol=1e-7)
    internal = present & (nodes["is_leaf"] == 0)
    np.testing.assert_allclose(nodes["gain"][internal], onodes["gain"][internal], rtol=1e-6, atol=1e-9)
    np.testing.assert_allclose(margin, omargin, rtol=RTOL, atol=ATOL)
    return st


def structural_invariants(nodes, n, d, lam, gamma):
    """Properties that hold at any size (used where the oracle cannot run)."""
    for t in range(nodes.shape[0]):
        tr = nodes[t]
        assert tr[0]["heap_id"] == 0 and tr[0]["count"] == n
        leaves = 0
        for k in np.where(tr["heap_id"] >= 0)[0]:
            nd = tr[k]
            assert int(np.floor(np.log2(k + 1))) <= d
            if nd["is_leaf"]:
                leaves += int(nd["count"])
                assert nd["weight"] == -nd["G"] / (nd["H"] + lam)
            else:
                hi, lo = tr[2 * k + 1], tr[2 * k + 2]
                assert hi["heap_id"] == 2 * k + 1 and lo["heap_id"] == 2 * k + 2
                assert hi["count"] + lo["count"] == nd["count"] and hi["count"] >= 1 and lo["count"] >= 1
                assert np.isclose(hi["G"] + lo["G"], nd["G"], rtol=1e-9, atol=1e-6)
                assert np.isclose(hi["H"] + lo["H"], nd["H"], rtol=1e-9, atol=1e-6)
                assert nd["gain"] > max(gamma, 0.0)
        assert leaves == n
