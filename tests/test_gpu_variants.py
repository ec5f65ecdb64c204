"""SURVEY §8(f3) and §8(f4) on the GPU (-m gpu), through the C ABI.

f3  RLE variants: the paper's "splitting RLE with decompression" (Fig. 6) must
    give the same trees as the direct split of the runs (Fig. 7) -- both build
    RLE(filter(root column)) -- and AUTO decides per attribute on entries/runs >= R (P:237,
    reading R21): low-cardinality attributes are compressed, the others stay plain.
f4  the dense representation: absent values filled (default 0) before the
    attribute lists are sorted; the oracle trains on the same filled matrix written out as CSR.
"""
import numpy as np
import pytest

from datagen import synth
from paper_conf_ipps_wenhkls18_b200 import gbdt

from parity import compare

pytestmark = pytest.mark.gpu


def _same(a, b):
    ma, ya = a
    mb, yb = b
    assert np.array_equal(ma.nodes().view(np.uint8), mb.nodes().view(np.uint8))
    assert np.array_equal(ya, yb)


# ------------------------------------------------------------------ f3: RLE split by decompression
@pytest.mark.parametrize("maker", [
    lambda: synth.c5(n=40000, T=3),
    lambda: synth.random_small(41, n=6000, m=6, nan_frac=0.25, n_distinct=12),
    lambda: synth.c4(seed=9, n=1500, m=2000, density=0.01, T=2),
    lambda: synth.random_small(42, n=8000, m=5, nan_frac=0.1, n_distinct=20, loss="logistic", d=8, T=2),
])
def test_rle_split_by_decompression_equals_direct(maker):
    p = maker()
    direct = gbdt.train_problem(p, rle="on")
    dec = gbdt.train_problem(p, rle="on", rle_split="decompress")
    _same(direct, dec)
    compare(p, dec[0].nodes(), dec[1])


# ------------------------------------------------------------------ f3: AUTO per attribute
def _mixed_cardinality(n=30000, seed=3):
    rng = np.random.default_rng(seed)
    X = np.empty((n, 6))
    X[:, 0] = rng.integers(0, 4, n)              # 4 distinct: compress
    X[:, 1] = rng.normal(size=n)                 # continuous: plain
    X[:, 2] = rng.normal(size=n)                 # continuous: plain
    X[:, 3] = rng.integers(0, 50, n)             # 50 distinct: compress
    X[:, 4] = np.round(rng.uniform(size=n), 1)   # 11 distinct: compress
    X[:, 5] = rng.normal(size=n)                 # continuous: plain
    y = (X[:, 0] + X[:, 1] + 0.3 * X[:, 3] / 10 + rng.normal(size=n) > 1.5).astype(np.float64)
    return synth.from_dense("mixed", X, y, dict(loss="logistic", max_depth=5, n_trees=3, lam=1.0, gamma=0.0,
                                                eta=0.3, base_margin=0.0))


def test_rle_auto_decides_per_attribute(monkeypatch):
    p = _mixed_cardinality()
    ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m, rle="auto", rle_min_ratio=2.0)
    k = ds.info(0)["n_shards"]
    groups = [(ds.info(s)["attr_begin"], ds.info(s)["attr_end"], ds.info(s)["runs"] > 0) for s in range(k)]
    assert groups == [(0, 1, True), (1, 3, False), (3, 5, True), (5, 6, False)], groups
    m_auto, y_auto = gbdt.train(ds, **{k2: v for k2, v in p.params.items()})
    compare(p, m_auto.nodes(), y_auto)                       # RLE shards split on their runs
    monkeypatch.setenv("GBDT_FUSED", "0")
    monkeypatch.setenv("GBDT_RUNSPLIT", "0")                 # per-entry scan of the runs:
    m_scan = gbdt.train(ds, **{k2: v for k2, v in p.params.items()})
    _same(m_scan, gbdt.train_problem(p))                     # trees as without RLE, bit for bit


def test_rle_auto_uniform_decision_keeps_one_shard():
    p = synth.c5(n=20000, T=1)                  # every attribute <= 64 distinct values
    ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m, rle="auto")
    assert ds.info(0)["n_shards"] == 1 and ds.info(0)["runs"] > 0


# ------------------------------------------------------------------ f4: dense representation
def _filled(p, fill):
    X = p.dense()
    X[np.isnan(X)] = fill
    return synth.from_dense(p.name + "-filled", X, p.labels, dict(p.params))


@pytest.mark.parametrize("fill", [0.0, -1.5])
@pytest.mark.parametrize("maker", [
    lambda: synth.c4(seed=12, n=2000, m=300, density=0.05, T=3),
    lambda: synth.random_small(13, n=4000, m=7, nan_frac=0.3, n_distinct=9, loss="squared", d=5, T=3),
])
def test_dense_representation_equals_filled_matrix(maker, fill):
    p = maker()
    model, margin = gbdt.train_problem(p, dense=True, dense_fill=fill)
    q = _filled(p, fill)
    compare(q, model.nodes(), margin)                        # the oracle on the explicitly filled CSR
    # prediction on the ORIGINAL sparse rows fills the absent values the same way
    pred = model.predict(p.indptr, p.indices, p.values, p.m)
    assert np.array_equal(pred, margin)


def test_dense_representation_of_dense_data_is_a_no_op():
    p = synth.c1(n=3000)
    _same(gbdt.train_problem(p), gbdt.train_problem(p, dense=True))
