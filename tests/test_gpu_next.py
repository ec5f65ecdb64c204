"""SURVEY §8(f) rows beyond the hot path, through the C ABI (-m gpu):

f1  SmartGD ablation (Fig. 9): smartgd_off recomputes every prediction by traversing
    all previous trees, with the same operations in the same order, so the model and the training
    margin must be bit-identical to the SmartGD run.
f4  user-defined loss hook ("users can define their own loss function"): a callback over
    device pointers.  A callback computing the paper's squared loss must reproduce the built-in
    squared-loss model; one computing the logistic loss is checked against the oracle.
"""
import ctypes as C

import numpy as np
import pytest

from datagen import synth
from paper_conf_ipps_wenhkls18_b200 import gbdt

from parity import compare

pytestmark = pytest.mark.gpu


def _same_model(a, b):
    na, nb = a.nodes(), b.nodes()
    assert na.tobytes() == nb.tobytes()


@pytest.mark.parametrize("maker", [
    lambda: synth.c1(n=3000),
    lambda: synth.random_small(4, n=2000, m=9, nan_frac=0.3, n_distinct=30, loss="logistic", d=5, T=4),
    lambda: synth.c4(seed=7, n=700, m=2500, density=0.01),
])
def test_smartgd_off_bit_identical(maker):
    p = maker()
    m_on, y_on = gbdt.train_problem(p)
    m_off, y_off = gbdt.train_problem(p, smartgd=False)
    _same_model(m_on, m_off)
    assert y_on.tobytes() == y_off.tobytes()


def test_smartgd_off_needs_rows():
    p = synth.c1(n=500)
    ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m)
    with pytest.raises(gbdt.GbdtError, match="E_STATE"):
        gbdt.train(ds, max_depth=3, n_trees=2, smartgd=False)


def _host_grad(kind):
    """A user loss over device pointers: copies yhat/labels to the host (cuda-python runtime),
    computes g, h in numpy with the paper's formulas and copies them back, synchronously."""
    from cuda.bindings import runtime as rt

    def fn(n, yh, y, g, h, stream):
        assert rt.cudaStreamSynchronize(stream)[0] == rt.cudaError_t.cudaSuccess
        Y = np.empty(n, np.float64)
        L = np.empty(n, np.float32)
        assert rt.cudaMemcpy(Y.ctypes.data, yh, 8 * n, rt.cudaMemcpyKind.cudaMemcpyDeviceToHost)[0] == 0
        assert rt.cudaMemcpy(L.ctypes.data, y, 4 * n, rt.cudaMemcpyKind.cudaMemcpyDeviceToHost)[0] == 0
        yy = L.astype(np.float64)
        if kind == "squared":  # g = 2(yhat - y), h = 2 (reading R6)
            G = 2.0 * (Y - yy)
            H = np.full(n, 2.0)
        else:  # cross-entropy, Eq. 1, reading R5
            p = 1.0 / (1.0 + np.exp(-Y))
            G = p - yy
            H = np.maximum(p * (1.0 - p), 1e-16)
        assert rt.cudaMemcpy(g, G.ctypes.data, 8 * n, rt.cudaMemcpyKind.cudaMemcpyHostToDevice)[0] == 0
        assert rt.cudaMemcpy(h, H.ctypes.data, 8 * n, rt.cudaMemcpyKind.cudaMemcpyHostToDevice)[0] == 0
    return fn


def test_custom_loss_squared_equals_builtin():
    p = synth.c1(n=3000)
    m_b, y_b = gbdt.train_problem(p)
    m_c, y_c = gbdt.train_problem(p, loss="custom", grad_fn=_host_grad("squared"))
    nb, nc = m_b.nodes(), m_c.nodes()
    for f in ("heap_id", "is_leaf", "attr", "default_left", "split_value", "count"):
        assert np.array_equal(nb[f], nc[f]), f
    np.testing.assert_allclose(nc["weight"], nb["weight"], rtol=1e-12, atol=1e-15)
    np.testing.assert_allclose(y_c, y_b, rtol=1e-12, atol=1e-15)


@pytest.mark.parametrize("maker", [
    lambda: synth.random_small(9, n=1500, m=6, nan_frac=0.25, n_distinct=25, loss="logistic", d=4, T=3),
    lambda: synth.c2(n=4000, T=5),
])
def test_custom_loss_logistic_against_oracle(maker):
    p = maker()
    model, margin = gbdt.train_problem(p, loss="custom", grad_fn=_host_grad("logistic"))
    compare(p, model.nodes(), margin)


def test_custom_loss_errors():
    p = synth.c1(n=300)
    ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m)
    with pytest.raises(gbdt.GbdtError, match="E_INVAL"):
        gbdt.train(ds, max_depth=2, n_trees=1, loss="custom")

    def bad(n, yh, y, g, h, stream):
        raise RuntimeError("user loss failed")
    with pytest.raises(gbdt.GbdtError, match="grad_fn failed"):
        gbdt.train(ds, max_depth=2, n_trees=1, loss="custom", grad_fn=bad)


@pytest.mark.parametrize("poison", ["nan_g", "inf_h", "neg_h"])
def test_custom_loss_rejects_invalid_derivatives(poison):
    """The callback's contract (gbdt.h: h >= 0 and finite) is checked before the sums use it."""
    from cuda.bindings import runtime as rt
    p = synth.c1(n=400)
    ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m)
    good = _host_grad("squared")

    def fn(n, yh, y, g, h, stream):
        good(n, yh, y, g, h, stream)
        H = np.empty(n, np.float64)
        G = np.empty(n, np.float64)
        assert rt.cudaMemcpy(G.ctypes.data, g, 8 * n, rt.cudaMemcpyKind.cudaMemcpyDeviceToHost)[0] == 0
        assert rt.cudaMemcpy(H.ctypes.data, h, 8 * n, rt.cudaMemcpyKind.cudaMemcpyDeviceToHost)[0] == 0
        if poison == "nan_g":
            G[7] = np.nan
        elif poison == "inf_h":
            H[3] = np.inf
        else:
            H[11] = -1.0
        assert rt.cudaMemcpy(g, G.ctypes.data, 8 * n, rt.cudaMemcpyKind.cudaMemcpyHostToDevice)[0] == 0
        assert rt.cudaMemcpy(h, H.ctypes.data, 8 * n, rt.cudaMemcpyKind.cudaMemcpyHostToDevice)[0] == 0
    with pytest.raises(gbdt.GbdtError, match="non-finite g or h"):
        gbdt.train(ds, max_depth=2, n_trees=1, loss="custom", grad_fn=fn)


@pytest.mark.parametrize("maker", [
    lambda: synth.c1(n=3000),
    lambda: synth.c4(seed=3, n=600, m=2000, density=0.01),
    lambda: synth.c5(n=20000, T=3),
])
def test_graph_replay_bit_identical(maker, monkeypatch):
    """the tree loop replayed as one CUDA graph per tree equals eager launches."""
    p = maker()
    monkeypatch.setenv("GBDT_GRAPH", "0")
    m_e, y_e = gbdt.train_problem(p)
    monkeypatch.setenv("GBDT_GRAPH", "1")
    m_g, y_g = gbdt.train_problem(p)
    _same_model(m_e, m_g)
    assert y_e.tobytes() == y_g.tobytes()
    compare(p, m_g.nodes(), y_g)


def _traverse(nodes, eta, base, X):
    """Host traversal of the model's trees (reading R11): present x >= split_value goes
    high (2k+1), missing follows default_left; y accumulated in tree order in fp64."""
    n = X.shape[0]
    out = np.empty(n)
    for i in range(n):
        y = base
        for t in range(nodes.shape[0]):
            T = nodes[t]
            k = 0
            while not T[k]["is_leaf"]:
                x = X[i, T[k]["attr"]]
                high = bool(T[k]["default_left"]) if np.isnan(x) else bool(np.float32(x) >= T[k]["split_value"])
                k = 2 * k + 1 if high else 2 * k + 2
            y = y + eta * T[k]["weight"]
        out[i] = y
    return out


@pytest.mark.parametrize("m_train", [6, 90])  # dense shared-memory kernel / CSR binary search
def test_predict_kernels_match_host_traversal(m_train):
    rng = np.random.default_rng(m_train)
    p = synth.random_small(21, n=400, m=m_train, nan_frac=0.2, n_distinct=12, loss="logistic", d=4, T=3)
    model, margin = gbdt.train_problem(p)
    # new rows: NaN, -0.0 and columns past the training n_cols (ignored = missing)
    n2, m2 = 300, m_train + 3
    X = rng.integers(0, 12, size=(n2, m2)).astype(np.float32) / 4 - 1.0
    X[rng.random((n2, m2)) < 0.25] = np.nan
    X[rng.random((n2, m2)) < 0.05] = -0.0
    mask = ~np.isnan(X) | (rng.random((n2, m2)) < 0.5)  # some NaNs stored explicitly, others absent
    indptr = np.concatenate([[0], np.cumsum(mask.sum(1))]).astype(np.int64)
    indices = np.nonzero(mask)[1].astype(np.int32)
    values = X[mask].astype(np.float32)
    got = model.predict(indptr, indices, values, m2)
    Xd = np.where(mask, X, np.nan)[:, :m_train]
    want = _traverse(model.nodes(), p.params.get("eta", 0.3), p.params.get("base_margin", 0.0), Xd)
    assert got.tobytes() == want.tobytes()
    # and the training rows reproduce the training margin
    assert np.array_equal(model.predict(p.indptr, p.indices, p.values, p.m), margin)


@pytest.mark.parametrize("maker", [lambda: synth.c1(n=2000), lambda: synth.c2(n=5000, T=4)])
def test_train_loss_per_tree(maker):
    """gbdt_model_train_loss: the mean training loss after 0 .. T trees (P:415-431 reports RMSE),
    against the loss of the oracle's prediction with the first k trees on the training rows."""
    from oracle import oracle
    p = maker()
    model, margin = gbdt.train_problem(p)
    L = model.train_loss()
    nodes = model.nodes()
    T = nodes.shape[0]
    assert L.shape == (T + 1,)
    y = p.labels.astype(np.float64)
    for k in range(T + 1):
        m = oracle.predict(nodes[:k], p.indptr, p.indices, p.values, eta=p.params["eta"]) if k else np.zeros(p.n)
        if p.params["loss"] == "squared":
            ref = np.mean((y - m) ** 2)
        else:
            ref = np.mean(np.maximum(m, 0) - y * m + np.log1p(np.exp(-np.abs(m))))
        assert L[k] == pytest.approx(ref, rel=1e-9), (k, L[k], ref)
    assert L[-1] < L[0]
