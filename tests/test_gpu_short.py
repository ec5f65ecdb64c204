"""Short-list path (levels.cu k_short_split / k_short_count / k_short_scatter / k_short_update) on the GPU (-m gpu).

Sparse attributes whose root list has at most 32 entries are split and partitioned a lane per entry,
32/W lists per warp, at levels 0-5; the chunk kernels take the other attributes.  The path keeps the
chunk kernels' arithmetic and association (k_sf_short's segmented scans, agg_short's present
totals), so trees and margins must be BIT-identical with the path on (default) and off
(GBDT_SHORT=0), and both match the oracle.  The cases cover the three gradient storage modes, new
leaves dropping entries (gamma), the hand-over to the chunk kernels below level 5 (depth 8), lists
of every length class around the batch widths, and attribute shards.
"""
import numpy as np
import pytest

from datagen import synth
from paper_conf_ipps_wenhkls18_b200 import gbdt

from parity import compare

pytestmark = pytest.mark.gpu


def _pair(monkeypatch, p, **kw):
    monkeypatch.setenv("GBDT_SHORT", "0")
    ref, ref_margin = gbdt.train_problem(p, **kw)
    monkeypatch.setenv("GBDT_SHORT", "1")
    model, margin = gbdt.train_problem(p, **kw)
    monkeypatch.delenv("GBDT_SHORT")
    return ref, ref_margin, model, margin


def _same(ref, ref_margin, model, margin):
    assert np.array_equal(model.nodes().view(np.uint8), ref.nodes().view(np.uint8))
    assert np.array_equal(margin.view(np.uint64), ref_margin.view(np.uint64))


def _fractional_labels(p):
    """logistic with labels in (0, 1): g and h both gathered (the kHGather storage mode)."""
    rng = np.random.Generator(np.random.PCG64(77))
    p.labels = rng.uniform(0.05, 0.95, p.n).astype(np.float32)
    return p


@pytest.mark.parametrize("name,maker,kw", [
    ("logistic", lambda: synth.c4(seed=9, n=1500, m=2000, density=0.01, T=3), {}),
    ("squared", lambda: synth.c4(seed=10, n=1500, m=2000, density=0.01, T=3), {"loss": "squared"}),
    ("h-gathered", lambda: _fractional_labels(synth.c4(seed=11, n=1500, m=2000, density=0.01, T=3)), {}),
    ("gamma-leaves", lambda: synth.c4(seed=12, n=3000, m=3000, density=0.01, T=3), {"gamma": 0.5}),
    ("depth8", lambda: synth.c4(seed=13, n=4000, m=3000, density=0.01, T=2), {"max_depth": 8}),
    ("c4b-shape", lambda: synth.c4(seed=14, n=8000, m=2500, density=0.004, T=2), {}),
])
def test_short_path_bit_identical_and_oracle(monkeypatch, name, maker, kw):
    p = maker()
    ref, ref_margin, model, margin = _pair(monkeypatch, p, **kw)
    _same(ref, ref_margin, model, margin)
    params = dict(p.params)
    params.update(kw)
    compare(p, model.nodes(), margin, params=params)


def test_short_path_length_classes(monkeypatch):
    """Every root length 1..40 (batch widths 1, 2, 4, 8, 16, 32 and the chunk path past 32), with
    repeated values so that runs end inside lists, and missing values everywhere."""
    rng = np.random.Generator(np.random.PCG64(5))
    n, m = 600, 400
    rows, cols, vals = [], [], []
    for a in range(m):
        L = 1 + a % 40
        r = rng.choice(n, size=L, replace=False)
        v = rng.integers(0, 6, L).astype(np.float32) / 3.0
        rows.append(r); cols.append(np.full(L, a)); vals.append(v)
    rows = np.concatenate(rows); cols = np.concatenate(cols); vals = np.concatenate(vals)
    o = np.lexsort((cols, rows))
    rows, cols, vals = rows[o], cols[o].astype(np.int32), vals[o]
    indptr = np.zeros(n + 1, np.int64)
    np.cumsum(np.bincount(rows, minlength=n), out=indptr[1:])
    y = (rng.uniform(0, 1, n) < 0.5).astype(np.float32)
    p = synth.Problem("lenclass", n, m, indptr, cols, vals, y, synth._params("logistic", 6, 3))
    ref, ref_margin, model, margin = _pair(monkeypatch, p)
    _same(ref, ref_margin, model, margin)
    compare(p, model.nodes(), margin)


def test_short_path_shards(monkeypatch):
    p = synth.c4(seed=15, n=1200, m=2500, density=0.01, T=2)
    ref, ref_margin, model, margin = _pair(monkeypatch, p, n_shards=4)
    _same(ref, ref_margin, model, margin)
    one, one_margin = gbdt.train_problem(p)
    _same(one, one_margin, model, margin)


# In-place short lists (depth <= 6, the default there): never partitioned, node index per entry
# updated in place, lanes sorted by node before the scans -- bit-identical to the partitioned short
# lists (GBDT_SHORT_INPLACE=0), including new leaves (0xff entries), shards and every gradient mode.
@pytest.mark.parametrize("name,maker,kw", [
    ("logistic", lambda: synth.c4(seed=21, n=2000, m=2500, density=0.01, T=3), {}),
    ("squared-gamma", lambda: synth.c4(seed=22, n=3000, m=3000, density=0.01, T=3), {"loss": "squared", "gamma": 0.5}),
    ("h-gathered", lambda: _fractional_labels(synth.c4(seed=23, n=1500, m=2000, density=0.01, T=2)), {}),
    ("shards", lambda: synth.c4(seed=24, n=2000, m=2500, density=0.01, T=2), {"n_shards": 4}),
])
def test_short_inplace_equals_partitioned(monkeypatch, name, maker, kw):
    p = maker()
    monkeypatch.setenv("GBDT_SHORT_INPLACE", "0")
    ref, ref_margin = gbdt.train_problem(p, **kw)
    monkeypatch.setenv("GBDT_SHORT_INPLACE", "1")
    model, margin = gbdt.train_problem(p, **kw)
    _same(ref, ref_margin, model, margin)
