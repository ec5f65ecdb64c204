"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times (-m gpu).

Tree-for-tree oracle parity at full size is tests/test_gpu_fullsize_parity.py.  This module
checks what holds at any size, on the bench's own 40-tree C3 run and across code paths:
  * structural invariants of every tree (counts, child totals, leaf weights, gains > gamma);
  * gbdt_predict on the training rows reproduces the training margin bit for bit;
  * C3: a 2-shard (loopback) run gives bit-identical trees.
"""
import numpy as np
import pytest

from paper_conf_ipps_wenhkls18_b200 import gbdt

from parity import full_problem, structural_invariants

pytestmark = pytest.mark.gpu


def _run(prob, T=1, **kw):
    P = dict(prob.params)
    P["n_trees"] = T
    P.update(kw)
    return gbdt.train_problem(prob, **P)


def test_full_size_c3_shards_bit_identical():
    prob = full_problem("C3")
    a, ma = _run(prob, T=1)
    b, mb = _run(prob, T=1, n_shards=2)
    assert np.array_equal(a.nodes().view(np.uint8), b.nodes().view(np.uint8))
    assert np.array_equal(ma, mb)


def test_full_size_c3_forty_trees_as_benched():
    """C3 at its full size and the bench's configuration (40 trees in one gbdt_train, one CUDA
    graph per tree): every tree satisfies the structural invariants, the first tree equals the
    one a 1-tree run builds, and prediction by traversal reproduces the SmartGD margin."""
    prob = full_problem("C3")
    model, margin = _run(prob, T=40)
    nodes = model.nodes()
    P = prob.params
    structural_invariants(nodes, prob.n, P["max_depth"], P["lam"], P["gamma"])
    one, _ = _run(prob, T=1)
    assert nodes[0].tobytes() == one.nodes()[0].tobytes()
    pred = gbdt.predict(model, prob.indptr, prob.indices, prob.values, prob.m)
    assert np.array_equal(pred, margin)
    assert np.isfinite(margin).all()
