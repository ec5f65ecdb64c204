"""Seeded synthetic inputs shaped like the paper's workloads (SURVEY.md §8(d) input recipe).

This module is shared by the oracle side and the CUDA side ONLY as an input source: it draws
random numbers and emits CSR matrices + labels. It contains none of the method's arithmetic
(no gradients, no sorting into attribute lists, no gains, no partitioning).

Every generator returns a :class:`Problem` with
  indptr  int64[n+1], indices int32[N], values float32[N]   (CSR, indices strictly increasing per row)
  labels  float32[n]
  params  dict(loss, max_depth, n_trees, lam, gamma, eta, base_margin)

Configs (BASELINE.json "configs"):
  C1 tiny dense 1,000 x 8 squared, d=3, T=2, lambda=1                       (PAPER.md none; oracle in seconds)
  C2 covtype-shaped dense 581,012 x 54 logistic, d=6, T=40
  C3 higgs-shaped dense 11,000,000 x 28 logistic, d=6, T=40
  C4 news20 / real-sim-shaped sparse, ~0.1% density, logistic, d=6, T=40
  C5 susy-shaped 5,000,000 x 18, <=64 distinct values per attribute (RLE)   (BASELINE.json)
`n` may be overridden to draw a smaller instance with the same per-row distribution.
"""
from __future__ import annotations

import dataclasses
import hashlib

import numpy as np


@dataclasses.dataclass
class Problem:
    name: str
    n: int
    m: int
    indptr: np.ndarray
    indices: np.ndarray
    values: np.ndarray
    labels: np.ndarray
    params: dict

    @property
    def nnz(self) -> int:
        return int(self.indptr[-1])

    def sha256(self) -> str:
        h = hashlib.sha256()
        for a in (self.indptr, self.indices, self.values, self.labels):
            h.update(np.ascontiguousarray(a).tobytes())
        return h.hexdigest()

    def dense(self) -> np.ndarray:
        """Dense float64 view with NaN for absent entries (tests only, small n)."""
        X = np.full((self.n, self.m), np.nan, dtype=np.float64)
        rows = np.repeat(np.arange(self.n), np.diff(self.indptr))
        X[rows, self.indices] = self.values
        return X


def _params(loss, d, T, lam=1.0, gamma=0.0, eta=0.3, base=0.0):
    return dict(loss=loss, max_depth=d, n_trees=T, lam=lam, gamma=gamma, eta=eta, base_margin=base)


def from_dense(name, X, y, params) -> Problem:
    """Dense matrix -> CSR with every entry stored (NaN entries are dropped = missing)."""
    X = np.asarray(X, dtype=np.float32)
    n, m = X.shape
    present = ~np.isnan(X)
    counts = present.sum(axis=1)
    indptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(counts, out=indptr[1:])
    cols = np.broadcast_to(np.arange(m, dtype=np.int32), (n, m))
    return Problem(name, n, m, indptr, cols[present].astype(np.int32, copy=False),
                   X[present].astype(np.float32, copy=False),
                   np.asarray(y, dtype=np.float32), params)


def from_dense_full(name, X, y, params) -> Problem:
    """Dense matrix without NaN -> CSR, built without boolean masking (fast for 300M entries)."""
    X = np.ascontiguousarray(X, dtype=np.float32)
    n, m = X.shape
    indptr = np.arange(0, n * m + 1, m, dtype=np.int64)
    indices = np.tile(np.arange(m, dtype=np.int32), n)
    return Problem(name, n, m, indptr, indices, X.reshape(-1), np.asarray(y, dtype=np.float32), params)


def _sigmoid(z):
    return 1.0 / (1.0 + np.exp(-z))


# --------------------------------------------------------------------------------------------
# Table I: x1={a3:0.1}, x2={a1:1.2,a3:0.1,a4:0.6}, x3={a1:0.5,a2:1.0}, x4={a1:1.2,a3:2.0}
# attributes a1..a4 -> columns 0..3; labels chosen in SURVEY.md Appendix A: y=(1,0,1,0).
# --------------------------------------------------------------------------------------------
def table1(loss="squared", d=2, T=2, lam=1.0, gamma=0.0, eta=1.0) -> Problem:
    indptr = np.array([0, 1, 4, 6, 8], dtype=np.int64)
    indices = np.array([2, 0, 2, 3, 0, 1, 0, 2], dtype=np.int32)
    values = np.array([0.1, 1.2, 0.1, 0.6, 0.5, 1.0, 1.2, 2.0], dtype=np.float32)
    labels = np.array([1, 0, 1, 0], dtype=np.float32)
    return Problem("table1", 4, 4, indptr, indices, values, labels, _params(loss, d, T, lam, gamma, eta))


def c1(seed=1, n=1000) -> Problem:
    rng = np.random.Generator(np.random.PCG64(seed))
    m = 8
    X = np.empty((n, m), dtype=np.float64)
    X[:, 0:5] = np.round(rng.uniform(0, 1, size=(n, 5)), 3)
    X[:, 5:7] = rng.integers(0, 5, size=(n, 2))
    X[:, 7] = X[:, 0]  # exact copy: exact gain ties must resolve to attribute 0
    y = np.sin(2 * np.pi * X[:, 0]) + X[:, 1] * X[:, 2] + 0.5 * (X[:, 5] >= 2) + rng.normal(0, 0.1, size=n)
    return from_dense_full("C1", X, y, _params("squared", 3, 2, 1.0, 0.0, 0.3))


def c2(seed=2, n=581012, T=40) -> Problem:
    """covtype-shaped: 10 integer attributes + 4-way and 40-way one-hot groups, all stored."""
    rng = np.random.Generator(np.random.PCG64(seed))
    m = 54
    X = np.zeros((n, m), dtype=np.float32)
    elev = np.clip(np.round(rng.normal(2959, 280, n)), 1859, 3858)
    X[:, 0] = elev
    X[:, 1] = rng.integers(0, 361, n)
    X[:, 2] = np.clip(np.round(rng.normal(14, 7.5, n)), 0, 66)
    X[:, 3] = np.clip(np.round(rng.exponential(270, n)), 0, 1397)
    X[:, 4] = np.clip(np.round(rng.normal(46, 58, n)), -173, 601)
    X[:, 5] = np.clip(np.round(rng.uniform(0, 7117, n) * rng.uniform(0.2, 1.0, n)), 0, 7117)
    X[:, 6] = np.clip(np.round(rng.normal(212, 27, n)), 0, 254)
    X[:, 7] = np.clip(np.round(rng.normal(223, 20, n)), 0, 254)
    X[:, 8] = np.clip(np.round(rng.normal(143, 38, n)), 0, 254)
    X[:, 9] = np.clip(np.round(rng.exponential(1980, n)), 0, 7173)
    wild = rng.choice(4, size=n, p=[0.45, 0.05, 0.44, 0.06])
    X[np.arange(n), 10 + wild] = 1.0
    zipf = 1.0 / np.arange(1, 41) ** 1.2
    soil = rng.choice(40, size=n, p=zipf / zipf.sum())
    X[np.arange(n), 14 + soil] = 1.0
    f = (0.004 * (elev - 2959) + 0.8 * (wild == 2) - 0.6 * (wild == 0) + 0.3 * (soil % 3 == 0)
         - 0.002 * (X[:, 3] - 270) + 0.2 * np.sin(X[:, 1] / 57.3) + rng.normal(0, 0.5, n))
    y = (rng.uniform(0, 1, n) < _sigmoid(f - np.median(f) + 0.0)).astype(np.float32)
    return from_dense_full("C2", X, y, _params("logistic", 6, T))


def c3(seed=3, n=11_000_000, T=40) -> Problem:
    """higgs-shaped: 21 low-level (6 pT-like, 5 eta-like, 6 phi-like, 4 b-tag with 3 values) + 7 mass-like."""
    rng = np.random.Generator(np.random.PCG64(seed))
    m = 28
    X = np.empty((n, m), dtype=np.float32)
    # column order follows HIGGS: lep(pt,eta,phi), met(mag,phi), 4 x jet(pt,eta,phi,btag), 7 high-level
    pt_cols = [0, 3, 5, 9, 13, 17]
    eta_cols = [1, 6, 10, 14, 18]
    phi_cols = [2, 4, 7, 11, 15, 19]
    btag_cols = [8, 12, 16, 20]
    for c in pt_cols:
        X[:, c] = rng.lognormal(0.0, 0.5, n)
    for c in eta_cols:
        X[:, c] = np.clip(rng.normal(0, 1, n), -2.5, 2.5)
    for c in phi_cols:
        X[:, c] = rng.uniform(-np.pi, np.pi, n)
    bvals = np.array([0.0, 1.0865, 2.1731], dtype=np.float32)
    for c in btag_cols:
        X[:, c] = bvals[rng.choice(3, size=n, p=[0.55, 0.15, 0.30])]
    for k in range(7):
        a, b = pt_cols[k % 6], pt_cols[(k + 2) % 6]
        X[:, 21 + k] = (np.sqrt(X[:, a] * X[:, b]) * rng.lognormal(0.0, 0.25, n)
                        * (1.0 + 0.1 * np.cos(X[:, phi_cols[k % 6]]))).astype(np.float32)
    f = (0.8 * np.log(X[:, 25]) - 0.5 * np.log(X[:, 26]) + 0.3 * (X[:, 8] > 1) + 0.2 * X[:, 0]
         - 0.15 * np.abs(X[:, 1]) + rng.normal(0, 0.8, n))
    y = (rng.uniform(0, 1, n) < _sigmoid(f - np.quantile(f, 0.47))).astype(np.float32)
    return from_dense_full("C3", X, y, _params("logistic", 6, T))


def c4(seed=41, n=19_954, m=1_355_191, density=0.001, T=40, name="C4a") -> Problem:
    """news20 / real-sim-shaped sparse: Zipf column popularity, lognormal row lengths, positive
    tf-idf-like values L2-normalised per row; absent entries are missing."""
    rng = np.random.Generator(np.random.PCG64(seed))
    mean_len = max(1.0, density * m)
    lens = np.maximum(1, np.round(rng.lognormal(np.log(mean_len) - 0.125, 0.5, n))).astype(np.int64)
    lens = np.minimum(lens, m)
    pop = (np.arange(m, dtype=np.float64) + 10.0) ** -1.1
    pop /= pop.sum()
    perm = rng.permutation(m)
    total = int(lens.sum())
    cols = perm[np.searchsorted(np.cumsum(pop), rng.uniform(0, 1, total), side="right").clip(0, m - 1)]
    rows = np.repeat(np.arange(n, dtype=np.int64), lens)
    key = np.unique(rows * m + cols)
    rows = (key // m).astype(np.int64)
    cols = (key % m).astype(np.int32)
    vals = rng.lognormal(0.0, 1.0, key.size)
    rn = np.sqrt(np.bincount(rows, weights=vals * vals, minlength=n))
    vals = (vals / rn[rows]).astype(np.float32)
    indptr = np.zeros(n + 1, dtype=np.int64)
    np.cumsum(np.bincount(rows, minlength=n), out=indptr[1:])
    w = rng.normal(0, 1, m) * (rng.uniform(0, 1, m) < 0.05)
    z = np.bincount(rows, weights=vals * w[cols], minlength=n) * 8.0 + rng.normal(0, 0.3, n)
    y = (rng.uniform(0, 1, n) < _sigmoid(z - np.median(z))).astype(np.float32)
    return Problem(name, n, m, indptr, cols, vals, y, _params("logistic", 6, T))


def c4b(seed=42, n=72_201, m=20_938, T=40) -> Problem:
    return c4(seed=seed, n=n, m=m, T=T, name="C4b")


def c4s(seed=43, n=20_000, m=400, T=40) -> Problem:
    """A SMALL sparse dataset (news20-shaped, 2 % density; 20k x 400 = 8M cells) for the dense-
    representation ablation of SURVEY §8(f4) (dense "if the data set is small").  Not a
    BASELINE.json config."""
    return c4(seed=seed, n=n, m=m, density=0.02, T=T, name="C4s")


def c5(seed=5, n=5_000_000, T=40, bins=64) -> Problem:
    """susy-shaped, low cardinality: continuous draws quantised into <=64 quantile bins per
    attribute, value = bin centre (fp32), so each root column has <=64 runs (RLE-heavy)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    m = 18
    Z = np.empty((n, m), dtype=np.float32)
    for c in range(8):
        Z[:, c] = rng.lognormal(0, 0.6, n) if c % 3 == 0 else rng.normal(0, 1, n)
    for c in range(8, 18):
        Z[:, c] = Z[:, (c * 5) % 8] * rng.lognormal(0, 0.3, n) + rng.normal(0, 0.2, n)
    f = 0.9 * Z[:, 0] - 0.7 * Z[:, 9] + 0.4 * Z[:, 3] * Z[:, 12] + rng.normal(0, 0.7, n)
    y = (rng.uniform(0, 1, n) < _sigmoid(f - np.quantile(f, 0.54))).astype(np.float32)
    X = np.empty_like(Z)
    qs = np.linspace(0, 1, bins + 1)
    for c in range(m):
        edges = np.quantile(Z[:, c], qs)
        edges[-1] = np.inf
        b = np.clip(np.searchsorted(edges, Z[:, c], side="right") - 1, 0, bins - 1)
        centre = np.empty(bins, dtype=np.float32)
        lo = np.quantile(Z[:, c], qs[:-1])
        hi = np.quantile(Z[:, c], qs[1:])
        centre[:] = (0.5 * (lo + hi)).astype(np.float32)
        X[:, c] = centre[b]
    return from_dense_full("C5", X, y, _params("logistic", 6, T))


def random_small(seed, n=16, m=4, nan_frac=0.2, n_distinct=5, loss="squared", d=3, T=2,
                 lam=1.0, gamma=0.0, eta=0.5) -> Problem:
    """Tiny random case with repeated values and NaN-missing entries (brute-force tests)."""
    rng = np.random.Generator(np.random.PCG64(seed))
    X = rng.integers(0, n_distinct, size=(n, m)).astype(np.float64) / 4.0 - 0.5
    X[rng.uniform(0, 1, size=(n, m)) < nan_frac] = np.nan
    if loss == "logistic":
        y = (rng.uniform(0, 1, n) < 0.5).astype(np.float32)
    else:
        y = rng.normal(0, 1, n)
    return from_dense(f"rand{seed}", X, y, _params(loss, d, T, lam, gamma, eta))


CONFIGS = {
    "C1": c1,
    "C2": c2,
    "C3": c3,
    "C4a": c4,
    "C4b": c4b,
    "C4s": c4s,
    "C5": c5,
}


def make(name: str, **kw) -> Problem:
    return CONFIGS[name](**kw)
