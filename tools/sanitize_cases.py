"""Small trainings covering every kernel family (dense, missing values, sparse short lists, RLE (split on runs) and
its decompression ablation, AUTO RLE, dense representation, loopback shards, deep trees,
SmartGD-off, the fused dense pass, prediction), for compute-sanitizer runs."""
import os
import sys

sys.path.insert(0, ".")
from datagen import synth  # noqa: E402
from paper_conf_ipps_wenhkls18_b200 import gbdt  # noqa: E402

cases = [
    ("C1", synth.c1(n=3000), {}),
    ("missing", synth.random_small(5, n=3000, m=6, nan_frac=0.3, n_distinct=40, loss="logistic", d=5, T=2), {}),
    ("sparse", synth.c4(seed=9, n=1500, m=4000, density=0.01, T=2), {}),
    ("rle", synth.c5(n=20000, T=2), {"rle": "on"}),
    ("shards", synth.c1(n=2000), {"n_shards": 4}),
    ("deep", synth.random_small(77, n=6000, m=6, nan_frac=0.0, n_distinct=400, loss="logistic", d=8, T=2), {}),
    ("smartgd_off", synth.c1(n=1000), {"smartgd": False}),
    ("rle_decompress", synth.c5(n=20000, T=2), {"rle": "on", "rle_split": "decompress"}),
    ("rle_auto", synth.c2(n=6000, T=2), {"rle": "auto"}),
    ("dense_repr", synth.c4(seed=12, n=800, m=200, density=0.05, T=2), {"dense": True}),
    ("fused", synth.c3(n=20000, T=2), {"_env": "GBDT_FUSED"}),
    # round 2: the split on runs (multi-run chunks, shards pipelined on streams, depth 8)
    ("rle_many_runs", synth.random_small(8, n=9000, m=5, nan_frac=0.0, n_distinct=3000), {"rle": "on"}),
    ("rle_shards", synth.c5(n=20000, T=2), {"rle": "on", "n_shards": 2}),
    ("rle_deep", synth.random_small(81, n=7000, m=4, nan_frac=0.0, n_distinct=200, loss="logistic", d=8, T=2),
     {"rle": "on"}),
    ("dense_shards", synth.c3(n=20000, T=2), {"n_shards": 4}),
]
for name, p, kw in cases:
    env = kw.pop("_env", None)
    if env:
        os.environ[env] = "1"
    model, margin = gbdt.train_problem(p, **kw)
    if env:
        del os.environ[env]
    model.predict(p.indptr, p.indices, p.values, p.m)
    print(name, "ok", flush=True)
