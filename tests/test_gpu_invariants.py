"""Kernel-level invariants of the level lists (-m gpu), checked on the lists the
library actually holds at a level (test hook GBDT_CAPTURE_LEVEL / gbdt_model_export_level):

  * every (node, attribute) segment is the root column of that attribute filtered by node
    membership, in the same order, bit for bit (the order-preserving partition, Fig. 2);
  * with RLE, the segment's runs are RLE of that filtered column (the direct run split, P:250,
    Fig. 7), both for the direct split and for the split-by-decompression ablation.

Node membership at the level is recomputed on the host by routing every instance through the
model's own splits above the level; the root columns come from the oracle's presort.
"""
import numpy as np
import pytest

from datagen import synth
from oracle import oracle
from paper_conf_ipps_wenhkls18_b200 import gbdt

pytestmark = pytest.mark.gpu


def _membership(X, tree, level):
    """Heap id of the node every instance is in at depth `level` (-1: it stopped in a leaf above)."""
    n = X.shape[0]
    h = np.zeros(n, np.int64)
    for _ in range(level):
        nd = tree[h.clip(0)]
        internal = (h >= 0) & (nd["is_leaf"] == 0) & (nd["heap_id"] >= 0)
        x = X[np.arange(n), nd["attr"].clip(0)]
        hi = np.where(np.isnan(x), nd["default_left"] == 1, x >= nd["split_value"])
        h = np.where(internal, np.where(hi, 2 * h + 1, 2 * h + 2), -1)
    return h


def _rle(vals):
    if vals.size == 0:
        return np.zeros(0, np.float32), np.zeros(0, np.int32)
    cut = np.flatnonzero(vals[1:] != vals[:-1]) + 1
    starts = np.concatenate([[0], cut])
    lens = np.diff(np.concatenate([starts, [vals.size]]))
    return vals[starts], lens.astype(np.int32)


CASES = [
    ("dense", lambda: synth.c3(n=30000, T=1), "off", "direct"),
    ("missing", lambda: synth.random_small(61, n=6000, m=6, nan_frac=0.3, n_distinct=25, loss="logistic", d=5, T=1),
     "off", "direct"),
    ("sparse", lambda: synth.c4(seed=7, n=3000, m=800, density=0.01, T=1), "off", "direct"),
    ("rle", lambda: synth.c5(n=30000, T=1), "on", "direct"),
    ("rle_missing", lambda: synth.random_small(62, n=6000, m=5, nan_frac=0.2, n_distinct=9, d=5, T=1), "on", "direct"),
    ("rle_decompress", lambda: synth.c5(n=30000, T=1), "on", "decompress"),
]


@pytest.mark.parametrize("level", [1, 2, 4])
@pytest.mark.parametrize("name,maker,rle,split", CASES, ids=[c[0] for c in CASES])
def test_level_segments_are_filtered_root_columns(name, maker, rle, split, level, monkeypatch):
    monkeypatch.setenv("GBDT_CAPTURE_LEVEL", str(level))
    p = maker()
    P = dict(p.params)
    P["n_trees"] = 1
    ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m, rle=rle, n_shards=2 if name == "dense" else 1)
    model, _ = gbdt.train(ds, rle_split=split, **{k: v for k, v in P.items()})
    tree = model.nodes()[0]
    X = p.dense()
    memb = _membership(X, tree, level)
    active = [h for h in range((1 << level) - 1, (1 << (level + 1)) - 1) if tree[h]["heap_id"] == h]
    col_ptr, oval, oins = oracle.presort(p.indptr, p.indices, p.values, p.n, p.m)
    nshards = ds.info(0)["n_shards"]
    checked = 0
    for s in range(nshards):
        cap = model.export_level(s)
        inf = ds.info(cap["shard"])
        a0, K = inf["attr_begin"], cap["K"]
        assert K == len(active)
        for a in range(cap["m"]):
            ga = a0 + a
            cv, ci = oval[col_ptr[ga]:col_ptr[ga + 1]], oins[col_ptr[ga]:col_ptr[ga + 1]]
            for j, h in enumerate(active):
                keep = memb[ci] == h
                ev, ei = cv[keep], ci[keep]
                s0, n = cap["seg_start"][a * K + j], cap["seg_cnt"][a * K + j]
                assert n == ev.size, (a, j, n, ev.size)
                assert np.array_equal(cap["ins"][s0:s0 + n], ei), (name, a, j)
                if rle == "off":  # with RLE the value list below the root is not maintained (values in runs)
                    assert np.array_equal(cap["val"][s0:s0 + n].view(np.uint32), ev.view(np.uint32)), (name, a, j)
                else:
                    r0, r1 = cap["seg_run"][a * K + j], cap["seg_run"][a * K + j + 1]
                    rv, rl = _rle(ev)
                    assert np.array_equal(cap["run_val"][r0:r1].view(np.uint32), rv.view(np.uint32)), (name, a, j)
                    assert np.array_equal(cap["run_len"][r0:r1], rl), (name, a, j)
                    assert np.array_equal(cap["run_pos"][r0:r1], s0 + np.cumsum(rl) - rl)
                checked += 1
    assert checked > 0
