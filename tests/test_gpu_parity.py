"""CUDA path vs the CPU oracle, element by element on the same seeded inputs (-m gpu).

Every call goes through the C ABI (libgbdt.so) via the ctypes binding.
"""
import numpy as np
import pytest

from datagen import synth
from oracle import oracle
from paper_conf_ipps_wenhkls18_b200 import gbdt

from parity import compare, structural_invariants

pytestmark = pytest.mark.gpu


def _train(prob, **kw):
    return gbdt.train_problem(prob, **kw)


# ------------------------------------------------------------------ a1 layout (bit-exact)
@pytest.mark.parametrize("maker", [
    lambda: synth.table1(),
    lambda: synth.c1(n=3000),
    lambda: synth.random_small(11, n=5000, m=7, nan_frac=0.3, n_distinct=40),
    lambda: synth.c4(seed=5, n=800, m=3000, density=0.01),
])
def test_layout_bit_exact(maker):
    p = maker()
    ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m)
    col_ptr, val, ins = ds.export_layout()
    ocp, oval, oins = oracle.presort(p.indptr, p.indices, p.values, p.n, p.m)
    assert np.array_equal(col_ptr, ocp)
    assert np.array_equal(val.view(np.uint32), oval.view(np.uint32))
    assert np.array_equal(ins, oins)


def test_layout_sharded_equals_unsharded():
    p = synth.c1(n=2000)
    base = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m).export_layout()
    for k in (2, 4, 8):
        ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m, n_shards=k)
        cols = []
        vals = []
        inss = []
        for s in range(k):
            cp, v, i = ds.export_layout(s)
            cols.append(np.diff(cp))
            vals.append(v)
            inss.append(i)
        assert np.array_equal(np.concatenate(cols), np.diff(base[0]))
        assert np.array_equal(np.concatenate(vals), base[1])
        assert np.array_equal(np.concatenate(inss), base[2])


# ------------------------------------------------------------------ worked example
def test_table1_appendix_a_on_gpu():
    p = synth.table1(loss="squared", d=2, T=2, lam=1.0, eta=1.0)
    model, margin = _train(p)
    nodes = model.nodes()
    compare(p, nodes, margin, allow_near_ties=False)
    assert nodes[0, 0]["attr"] == 0 and nodes[0, 0]["split_value"] == np.float32(1.2)
    np.testing.assert_allclose(margin, [0.96, 0.0, 0.96, 0.0], rtol=1e-12, atol=1e-15)


# ------------------------------------------------------------------ C1 (full config) and friends
def test_c1_full_config_exact():
    p = synth.c1()
    model, margin = _train(p)
    nodes = model.nodes()
    st = compare(p, nodes, margin, allow_near_ties=False)
    assert st["exact"] > 0
    assert not np.any(nodes["attr"] == 7)  # a7 duplicates a0: exact ties resolve to a0


@pytest.mark.parametrize("seed", range(8))
@pytest.mark.parametrize("loss", ["squared", "logistic"])
def test_random_missing_values(seed, loss):
    p = synth.random_small(seed + 100, n=200 + 37 * seed, m=3 + seed % 5, nan_frac=0.3,
                           n_distinct=3 + 2 * seed, loss=loss, d=4, T=3, lam=1.0,
                           gamma=0.02 if seed % 3 == 2 else 0.0, eta=0.4)
    model, margin = _train(p)
    compare(p, model.nodes(), margin)


@pytest.mark.parametrize("maker,T", [
    (lambda: synth.c2(n=20000, T=4), 4),
    (lambda: synth.c3(n=40000, T=3), 3),
    (lambda: synth.c5(n=30000, T=3), 3),
])
def test_shaped_subsamples(maker, T):
    p = maker()
    model, margin = _train(p)
    nodes = model.nodes()
    compare(p, nodes, margin)
    structural_invariants(nodes, p.n, p.params["max_depth"], p.params["lam"], p.params["gamma"])


def test_sparse_many_segments():
    p = synth.c4(seed=9, n=1500, m=4000, density=0.01, T=3)
    model, margin = _train(p)
    compare(p, model.nodes(), margin)


def test_multi_tile_ragged():
    # columns of 2048*k + ragged tails; exercises the Fenwick look-back across many tiles
    p = synth.random_small(77, n=2048 * 9 + 123, m=3, nan_frac=0.0, n_distinct=5000, loss="logistic",
                           d=5, T=2)
    model, margin = _train(p)
    compare(p, model.nodes(), margin)


# ------------------------------------------------------------------ edge cases
def test_constant_labels_no_split():
    p = synth.c1(n=500)
    p.labels[:] = 0.25
    model, margin = _train(p, eta=1.0, lam=1.0)
    nodes = model.nodes()
    # g == 0 everywhere -> every gain is exactly 0 -> no split (strict >)
    assert nodes[0, 0]["is_leaf"] == 1
    compare(p, nodes, margin, params=dict(eta=1.0), allow_near_ties=False)


def test_constant_and_missing_columns():
    X = np.random.default_rng(1).normal(size=(300, 4))
    X[:, 1] = 3.0
    X[:, 2] = np.nan
    X[::7, 3] = np.nan
    y = X[:, 0] + (np.nan_to_num(X[:, 3]) > 0)
    p = synth.from_dense("edge", X, y, dict(loss="squared", max_depth=3, n_trees=2, lam=1.0, gamma=0.0,
                                             eta=0.5, base_margin=0.0))
    model, margin = _train(p)
    compare(p, model.nodes(), margin)


def test_single_row_and_depth_one():
    p = synth.c1(n=1)
    model, margin = _train(p)
    compare(p, model.nodes(), margin)
    q = synth.c1(n=700)
    model, margin = _train(q, max_depth=1, n_trees=3)
    compare(q, model.nodes(), margin, params=dict(max_depth=1, n_trees=3))


def test_gamma_blocks_splits():
    p = synth.c1(n=700)
    model, margin = _train(p, gamma=1e9)
    nodes = model.nodes()
    assert np.all(nodes[:, 0]["is_leaf"] == 1)
    compare(p, nodes, margin, params=dict(gamma=1e9))


# ------------------------------------------------------------------ prediction
def test_predict_reproduces_training_margin_and_oracle():
    p = synth.random_small(5, n=3000, m=6, nan_frac=0.2, n_distinct=50, loss="logistic", d=5, T=4)
    model, margin = _train(p)
    pred = model.predict(p.indptr, p.indices, p.values, p.m)
    assert np.array_equal(pred, margin)
    opred = oracle.predict(_as_oracle(model.nodes()), p.indptr, p.indices, p.values, eta=p.params["eta"])
    assert np.array_equal(pred, opred)  # same trees, same op order -> bit-identical
    prob = gbdt.predict(model, p.indptr, p.indices, p.values, p.m, output_margin=False)
    np.testing.assert_allclose(prob, 1 / (1 + np.exp(-margin)), rtol=1e-15)


def _as_oracle(nodes):
    out = np.zeros(nodes.shape, oracle.NODE_DTYPE)
    for f in oracle.NODE_DTYPE.names:
        if f in nodes.dtype.names:
            out[f] = nodes[f]
    return out


# ------------------------------------------------------------------ sharding (loopback, 1 GPU)
@pytest.mark.parametrize("k", [2, 4, 8])
def test_loopback_shards_bit_identical(k):
    p = synth.c2(n=12000, T=3)
    ref_model, ref_margin = _train(p)
    ref = ref_model.nodes()
    model, margin = _train(p, n_shards=k)
    nodes = model.nodes()
    assert np.array_equal(nodes.view(np.uint8), ref.view(np.uint8))
    assert np.array_equal(margin, ref_margin)


def test_loopback_shards_sparse_missing():
    p = synth.c4(seed=3, n=1200, m=2500, density=0.01, T=2)
    ref_model, ref_margin = _train(p)
    model, margin = _train(p, n_shards=4)
    assert np.array_equal(model.nodes().view(np.uint8), ref_model.nodes().view(np.uint8))
    assert np.array_equal(margin, ref_margin)


def test_deterministic_across_runs():
    p = synth.c3(n=30000, T=2)
    a, ma = _train(p)
    b, mb = _train(p)
    assert np.array_equal(a.nodes().view(np.uint8), b.nodes().view(np.uint8))
    assert np.array_equal(ma, mb)


# ------------------------------------------------------------------ a8 RLE: direct split
# The RLE path reads values from the runs and splits the runs themselves (no decompression in HBM).
# With its per-entry scan (GBDT_RUNSPLIT=0) it sees the same entry streams as the plain lists, so
# its trees and margins must be bit-identical to the plain level-by-level path (GBDT_FUSED=0: dense
# data otherwise takes the fused pass of fused.cu, whose sums associate differently; GBDT_SHORT=0:
# the same for the short-list path), and both match the oracle.  The split on runs (the default
# for dense RLE data, k_run_split) is tested against the oracle below.
@pytest.mark.parametrize("maker", [
    lambda: synth.c5(n=40000, T=3),
    lambda: synth.table1(),
    lambda: synth.random_small(7, n=6000, m=6, nan_frac=0.25, n_distinct=12),
    lambda: synth.random_small(8, n=9000, m=5, nan_frac=0.0, n_distinct=3000),
    lambda: synth.c4(seed=9, n=1500, m=2000, density=0.01, T=2),
    lambda: synth.c1(n=5000),
])
def test_rle_direct_split_bit_identical(maker, monkeypatch):
    p = maker()
    monkeypatch.setenv("GBDT_FUSED", "0")
    monkeypatch.setenv("GBDT_RUNSPLIT", "0")
    # plain lists route short sparse attributes through the short path (levels.cu k_short_*), whose
    # prefix sums associate in list order; the RLE path keeps the chunk kernels throughout
    monkeypatch.setenv("GBDT_SHORT", "0")
    ref_model, ref_margin = _train(p)
    model, margin = _train(p, rle="on")
    assert np.array_equal(model.nodes().view(np.uint8), ref_model.nodes().view(np.uint8))
    assert np.array_equal(margin, ref_margin)


def test_rle_c5_against_oracle():
    p = synth.c5(n=20000, T=2)
    model, margin = _train(p, rle="on")
    compare(p, model.nodes(), margin)


@pytest.mark.parametrize("k", [2, 4])
def test_rle_with_shards(k, monkeypatch):
    p = synth.c5(n=30000, T=2)
    monkeypatch.setenv("GBDT_FUSED", "0")
    monkeypatch.setenv("GBDT_RUNSPLIT", "0")
    ref_model, ref_margin = _train(p)
    model, margin = _train(p, rle="on", n_shards=k)
    assert np.array_equal(model.nodes().view(np.uint8), ref_model.nodes().view(np.uint8))
    assert np.array_equal(margin, ref_margin)


# ------------------------------------------------------------------ a4-a6 RLE: split on runs
# Dense RLE data: every run's (G, H) is an exact fixed-point total of its chunk partials and the
# candidates are the run ends, so the result is oracle-equal and independent of the sharding.
# Cases: C5-shaped (<= 64 values), Table I, high cardinality (many runs per segment: the 32-run
# steps and their carry), squared and logistic, depth 8 (more than 32 nodes: global records),
# general labels (h gathered, hmode 2), C2-shaped (one-hot and integer columns).
@pytest.mark.parametrize("maker", [
    lambda: synth.c5(n=40000, T=3),
    lambda: synth.table1(),
    lambda: synth.random_small(8, n=9000, m=5, nan_frac=0.0, n_distinct=3000),
    lambda: synth.random_small(81, n=7000, m=4, nan_frac=0.0, n_distinct=200, loss="logistic", d=8, T=2),
    lambda: synth.c1(n=5000),
    lambda: synth.c2(n=30000, T=3),
])
def test_rle_run_split_against_oracle(maker):
    p = maker()
    model, margin = _train(p, rle="on")
    compare(p, model.nodes(), margin)


def test_rle_run_split_general_labels():
    """Logistic loss with labels outside {0, 1}: h is gathered per entry (hmode 2)."""
    p = synth.c5(n=20000, T=2)
    p.labels = (p.labels * 0.8 + 0.1).astype(np.float32)
    model, margin = _train(p, rle="on")
    compare(p, model.nodes(), margin)


@pytest.mark.parametrize("k", [2, 4])
def test_rle_run_split_shards_bit_identical(k):
    p = synth.c5(n=30000, T=3)
    ref_model, ref_margin = _train(p, rle="on")
    model, margin = _train(p, rle="on", n_shards=k)
    assert np.array_equal(model.nodes().view(np.uint8), ref_model.nodes().view(np.uint8))
    assert np.array_equal(margin, ref_margin)
    compare(p, model.nodes(), margin)


def test_rle_run_split_equals_entry_scan_structure(monkeypatch):
    """The split on runs and the per-entry scan of the same runs choose the same splits (their
    sums associate differently, so weights agree to rounding)."""
    p = synth.c5(n=50000, T=3)
    model, margin = _train(p, rle="on")
    monkeypatch.setenv("GBDT_RUNSPLIT", "0")
    ref_model, ref_margin = _train(p, rle="on")
    a, b = model.nodes(), ref_model.nodes()
    for f in ("heap_id", "is_leaf", "attr", "default_left", "count", "split_value"):
        assert np.array_equal(a[f], b[f]), f
    np.testing.assert_allclose(a["weight"], b["weight"], rtol=1e-9, atol=1e-12)
    np.testing.assert_allclose(margin, ref_margin, rtol=1e-9, atol=1e-12)


def test_rle_export_matches_oracle_encoding():
    p = synth.c5(n=20000, T=1)
    ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m, rle="on")
    run_ptr, rv, rl = ds.export_rle()
    ocp, oval, _ = oracle.presort(p.indptr, p.indices, p.values, p.n, p.m)
    for a in range(p.m):
        orv, orl = oracle.rle_encode(oval[ocp[a]:ocp[a + 1]])
        assert np.array_equal(rv[run_ptr[a]:run_ptr[a + 1]].view(np.uint32), orv.view(np.uint32))
        assert np.array_equal(rl[run_ptr[a]:run_ptr[a + 1]], orl)
    assert run_ptr[-1] == rv.size


# ------------------------------------------------------------------ path boundaries (round 1b)
@pytest.mark.parametrize("n", [31, 32, 33, 255, 256, 257, 511, 513])
def test_chunk_boundaries_dense_deep(n):
    """Dense lists whose lengths straddle one warp (32, the short-chunk path) and one chunk (256);
    depth 6 so that late levels have up to 32 segments per list and chunks that cross segments
    (the scatter's per-entry aggregate path and k_desc's head/count flags)."""
    p = synth.random_small(300 + n, n=n, m=5, nan_frac=0.0, n_distinct=max(3, n // 3), loss="logistic",
                           d=6, T=3, eta=0.5)
    model, margin = _train(p)
    compare(p, model.nodes(), margin)


@pytest.mark.parametrize("seed", range(3))
def test_sparse_lists_around_32_entries(seed):
    """Sparse attribute lists of ~25-40 entries with missing values: both the short-chunk split
    path (<= 32) and the general one (> 32) on the same level, up to 32 nodes per level."""
    p = synth.c4(seed=40 + seed, n=3000, m=120, density=0.011, T=2)
    p.params["max_depth"] = 6
    model, margin = _train(p)
    compare(p, model.nodes(), margin)


def test_sparse_many_chunks_batched_split():
    """More chunks than 32 x the split kernels' warps (~189 k lists, most <= 32 entries, a Zipf head
    of lists up to ~7.8 k entries, missing values): k_sf_short and k_sf_gen test 32 descriptors
    per warp step only in this regime (and in the bench's C4a), so it needs a case of its own."""
    p = synth.c4(seed=50, n=8000, m=240_000, density=0.0015, T=2)
    p.params["max_depth"] = 6
    model, margin = _train(p)
    compare(p, model.nodes(), margin)
    structural_invariants(model.nodes(), p.n, 6, p.params["lam"], p.params["gamma"])


def test_scatter_aggregates_match_chunk_agg():
    """The next-level chunk aggregates accumulated by the scatter (data without missing values)
    and those k_chunk_agg computes (the same lists with one NaN column, which routes every level
    through k_chunk_agg) give trees that both match the oracle."""
    base = synth.random_small(909, n=6000, m=4, nan_frac=0.0, n_distinct=2000, loss="logistic", d=6, T=3)
    model, margin = _train(base)
    compare(base, model.nodes(), margin)
    X = np.full((base.n, base.m + 1), np.nan, np.float32)
    dense = np.zeros((base.n, base.m), np.float32)
    for i in range(base.n):
        cols = base.indices[base.indptr[i]:base.indptr[i + 1]]
        dense[i, cols] = base.values[base.indptr[i]:base.indptr[i + 1]]
    X[:, :base.m] = dense
    X[::7, base.m] = 1.0  # a sparse extra column makes the dataset "has missing"
    q = synth.from_dense("agg_missing", X, base.labels, dict(base.params))
    model2, margin2 = _train(q)
    compare(q, model2.nodes(), margin2)


def test_all_entries_missing_and_empty_rows():
    """Degenerate inputs: no stored entry at all (every value missing) gives single-leaf
    trees; rows without entries next to full rows still split on the present values."""
    P = dict(loss="squared", max_depth=3, n_trees=2, lam=1.0, gamma=0.0, eta=0.5, base_margin=0.0)
    X = np.full((50, 3), np.nan)
    y = np.linspace(-1, 1, 50)
    p = synth.from_dense("all-missing", X, y, P)
    assert p.nnz == 0
    model, margin = _train(p)
    nodes = model.nodes()
    assert (nodes["is_leaf"][:, 0] == 1).all() and (nodes["heap_id"][:, 1:] == -1).all()
    compare(p, nodes, margin)
    X = np.random.default_rng(3).normal(size=(200, 3))
    X[::3] = np.nan  # a third of the rows are empty
    p = synth.from_dense("empty-rows", X, np.nan_to_num(X[:, 1]), P)
    model, margin = _train(p)
    compare(p, model.nodes(), margin)


@pytest.mark.parametrize("maker", [
    lambda: synth.random_small(77, n=6000, m=6, nan_frac=0.0, n_distinct=400, loss="logistic", d=8, T=2),
    lambda: synth.random_small(78, n=5000, m=5, nan_frac=0.25, n_distinct=60, loss="squared", d=9, T=2),
    lambda: synth.c4(seed=13, n=3000, m=1500, density=0.02, T=2),
])
def test_deep_trees_more_than_32_nodes_per_level(maker):
    """Depth >= 7: more than 32 active nodes per level, so node bests go through the global record
    list (post_record, k_pick_tie/k_pick_best) and the scatter finds segments without the per-warp
    table -- the paths depth-6 configs never take."""
    p = maker()
    if p.name.startswith("C4"):
        p.params["max_depth"] = 8
    model, margin = _train(p)
    compare(p, model.nodes(), margin, params=p.params)


def test_deep_trees_rle_bit_identical(monkeypatch):
    """RLE run tables with more than 32 nodes per level (depth 8) equal the plain path."""
    p = synth.random_small(79, n=8000, m=5, nan_frac=0.1, n_distinct=20, loss="logistic", d=8, T=2)
    monkeypatch.setenv("GBDT_FUSED", "0")
    ref_model, ref_margin = _train(p)
    model, margin = _train(p, rle="on")
    assert np.array_equal(model.nodes().view(np.uint8), ref_model.nodes().view(np.uint8))
    assert np.array_equal(margin, ref_margin)
    compare(p, model.nodes(), margin)


# ------------------------------------------------------------------ fused dense levels (fused.cu)
# Dense data below the root takes one pass per level (partition of level l + split find of level
# l+1).  Against the oracle on shapes that exercise its tile machinery: many tiles per segment
# (look-back chains), segments ending inside tiles, tiles holding several segments at depth 7-8
# (up to 64 parent nodes), long runs of equal values crossing tiles (C5/C2-shaped), both losses,
# and the non-writing last pass.
@pytest.mark.parametrize("maker", [
    lambda: synth.c3(n=60000, T=3),
    lambda: synth.c5(n=50000, T=3),
    lambda: synth.c2(n=30000, T=4),
    lambda: synth.random_small(31, n=20000, m=4, nan_frac=0.0, n_distinct=7, loss="squared", d=8, T=2),
    lambda: synth.random_small(32, n=12000, m=3, nan_frac=0.0, n_distinct=5000, loss="logistic", d=7, T=2),
    lambda: synth.random_small(33, n=2049, m=3, nan_frac=0.0, n_distinct=2, loss="squared", d=2, T=3),
])
def test_fused_dense_against_oracle(maker, monkeypatch):
    monkeypatch.setenv("GBDT_FUSED", "1")
    p = maker()
    model, margin = _train(p)
    compare(p, model.nodes(), margin)


@pytest.mark.parametrize("k", [2, 4])
def test_fused_shards_bit_identical(k, monkeypatch):
    monkeypatch.setenv("GBDT_FUSED", "1")
    p = synth.c3(n=50000, T=2)
    a, ma = _train(p)
    b, mb = _train(p, n_shards=k)
    assert np.array_equal(a.nodes().view(np.uint8), b.nodes().view(np.uint8))
    assert np.array_equal(ma, mb)


def test_fused_equals_level_by_level_up_to_rounding(monkeypatch):
    p = synth.c3(n=40000, T=3)
    monkeypatch.setenv("GBDT_FUSED", "1")
    a, ma = _train(p)
    monkeypatch.setenv("GBDT_FUSED", "0")
    b, mb = _train(p)
    na, nb = a.nodes(), b.nodes()
    for f in ("heap_id", "is_leaf", "attr", "default_left", "split_value", "count"):
        assert np.array_equal(na[f], nb[f]), f
    np.testing.assert_allclose(na["weight"], nb["weight"], rtol=1e-10, atol=1e-14)
    np.testing.assert_allclose(ma, mb, rtol=1e-10, atol=1e-14)


# ------------------------------------------------------------------ P:116 edge values, CART
# Values as gbdt.h states them ("missing values"): NaN stored in the CSR is missing, -0.0 is
# +0.0, +-Inf are ordinary values; each case against the oracle (which reads the same CSR bytes).
def _edge_problem(kind, seed=17, n=3000, m=5, loss="logistic"):
    rng = np.random.default_rng(seed)
    X = rng.integers(-3, 4, size=(n, m)).astype(np.float64)
    if kind == "nan":
        X[rng.uniform(size=X.shape) < 0.2] = np.nan       # stored NaN entries (from_dense drops them)
    elif kind == "negzero":
        X[X == 0] = -0.0
        X[:, 0] = np.where(rng.uniform(size=n) < 0.5, -0.0, 0.0)  # a column of +-0 only
    elif kind == "inf":
        X[rng.uniform(size=X.shape) < 0.1] = np.inf
        X[rng.uniform(size=X.shape) < 0.1] = -np.inf
    Xf = np.nan_to_num(X, nan=0.0, posinf=5.0, neginf=-5.0)
    y = (np.sin(Xf[:, 1]) + 0.3 * rng.normal(size=n) > 0).astype(np.float64) if loss == "logistic" else \
        Xf[:, 2] + rng.normal(size=n)
    p = synth.from_dense(kind, X, y,
                         dict(loss=loss, max_depth=4, n_trees=3, lam=1.0, gamma=0.0, eta=0.3, base_margin=0.0))
    if kind == "nan":  # store the NaNs explicitly in the CSR (not dropped): the library must treat them as missing
        indptr = np.arange(0, n * m + 1, m, dtype=np.int64)
        p = synth.Problem(kind, n, m, indptr, np.tile(np.arange(m, dtype=np.int32), n), X.reshape(-1).astype(np.float32),
                          p.labels, p.params)
    return p


@pytest.mark.parametrize("kind", ["nan", "negzero", "inf"])
def test_edge_values_against_oracle(kind):
    p = _edge_problem(kind)
    if kind == "nan":
        assert np.isnan(p.values).any()
    if kind == "negzero":
        assert np.signbit(p.values[p.values == 0]).any()
    if kind == "inf":
        assert np.isinf(p.values).any()
    model, margin = _train(p)
    compare(p, model.nodes(), margin)


def test_lambda0_squared_is_cart_on_gpu():
    """Squared loss, lambda = 0, eta = 1, one tree: the GPU tree is scikit-learn's CART tree
    (same leaf partition, leaf value = mean target), a library routine the method reduces to."""
    from sklearn.tree import DecisionTreeRegressor
    rng = np.random.default_rng(4)
    n, m, d = 2000, 6, 4
    X = rng.uniform(-1, 1, size=(n, m)).astype(np.float32).astype(np.float64)
    y = np.sin(3 * X[:, 0]) + X[:, 1] * X[:, 2] + 0.1 * rng.normal(size=n)
    p = synth.from_dense("cart", X, y, dict(loss="squared", max_depth=d, n_trees=1, lam=0.0, gamma=0.0,
                                            eta=1.0, base_margin=0.0))
    model, margin = _train(p)
    sk = DecisionTreeRegressor(max_depth=d, random_state=0).fit(X.astype(np.float32), p.labels.astype(np.float64))
    leaves_sk = sk.apply(X.astype(np.float32))
    groups_sk = {frozenset(np.where(leaves_sk == l)[0]) for l in np.unique(leaves_sk)}
    groups_gpu = {frozenset(np.where(margin == v)[0]) for v in np.unique(margin)}
    assert groups_sk == groups_gpu
    np.testing.assert_allclose(margin, sk.predict(X.astype(np.float32)), rtol=0, atol=1e-9)


# ------------------------------------------------------------------ near-ties decided exactly (no follow mode)
# Two candidates of one chunk whose Eq. 2 gains differ by ~1e-9 relative (far below the 1e-6 band
# follow mode would forgive, far above the ~1e-15 ranking error of the in-chunk scores, DESIGN.md
# I3): the CUDA path must pick the exact maximiser the oracle picks, with no follow mode.
@pytest.mark.parametrize("delta", [3e-7, -3e-7])
@pytest.mark.parametrize("fused", ["0", "1"])
def test_close_candidates_in_one_chunk_pick_the_exact_best(delta, fused, monkeypatch):
    monkeypatch.setenv("GBDT_FUSED", fused)
    n = 200
    x = np.arange(n, dtype=np.float64)
    y = np.where((x < 60) | (x >= 140), 1.0, -1.0)
    y[0] += delta                      # breaks the symmetry of the splits at 60 and at 140
    X = np.stack([x, np.zeros(n)], axis=1)  # a second constant column (no candidate)
    for depth in (1, 2):
        p = synth.from_dense("near", X, y, dict(loss="squared", max_depth=depth, n_trees=1, lam=1.0, gamma=0.0,
                                                eta=1.0, base_margin=0.0))
        on, om, _ = oracle.train(p)
        model, margin = _train(p)
        nodes = model.nodes()
        g0, g1 = oracle.gain(*_two(p, 60)), oracle.gain(*_two(p, 140))
        rel = abs(g0 - g1) / max(g0, g1)
        assert 1e-12 < rel < 1e-7, rel
        for f in ("heap_id", "is_leaf", "attr", "split_value", "default_left", "count"):
            assert np.array_equal(nodes[f], on[f]), (f, nodes[f][0], on[f][0])
        np.testing.assert_allclose(margin, om, rtol=1e-12, atol=1e-12)


def _two(p, cut):
    """(GL, HL, G, H, lambda) of the split 'x >= cut' at the root, squared loss at yhat = 0."""
    g = -2.0 * p.labels.astype(np.float64)
    X = p.dense()
    hi = X[:, 0] >= cut
    return float(g[hi].sum()), 2.0 * float(hi.sum()), float(g.sum()), 2.0 * p.n, 1.0
