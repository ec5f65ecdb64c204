"""Tree-for-tree parity at BASELINE.json's FULL sizes (north_star acceptance; "without
approximation", "trees are identical"), in the launch configuration bench.py times (one
gbdt_train, one CUDA graph per tree).  -m gpu.

For every config the CUDA path trains the first K trees of the benched run; the CPU oracle then
trains the same K trees on the same full rows in follow mode, and `parity.check`
compares every node (structure exact up to the 1e-6 near-tie band, weights / margins 1e-5).

  C2  581,012 x 54     all 40 trees
  C4b 72,201 x 20,938  all 40 trees
  C4a 19,954 x 1.36M   first 5 trees
  C5  5M x 18          first 5 trees, RLE off and RLE on (each against the oracle)
  C3  11M x 28         first K=2 trees (the oracle needs ~1 min per full C3 tree on one core)

The oracle runs are single-threaded and independent, so they run concurrently in a thread pool
(ctypes drops the GIL); each thread's presort and per-tree wall times are written to
gpurun_out/oracle_fullsize.json (the measured oracle cost at full size, cited by bench.py's
cpu_baseline and DESIGN.md), with the host's core count and CPU model.
"""
import concurrent.futures as cf
import json
import os
import platform
import time

import numpy as np
import pytest

from oracle import oracle
from paper_conf_ipps_wenhkls18_b200 import gbdt

from parity import check, full_problem

pytestmark = pytest.mark.gpu

TREES = {"C3": 2, "C2": 40, "C5": 5, "C4a": 5, "C4b": 40}
ORDER = ["C3", "C5", "C2", "C4a", "C4b"]            # longest oracle run first


def _cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return platform.processor()


def _oracle_job(prob, nodes, T):
    t0 = time.perf_counter()
    out = oracle.train(prob, params=dict(n_trees=T), follow=nodes)
    wall = time.perf_counter() - t0
    presort, trees = oracle.last_timings()
    return out, dict(wall_s=wall, presort_s=presort, tree_s=trees, n=prob.n, m=prob.m, nnz=prob.nnz,
                     trees=T, stats=out[2])


@pytest.fixture(scope="module")
def runs():
    pool = cf.ThreadPoolExecutor(max_workers=len(ORDER) + 1)
    res = {}
    for name in ORDER:
        prob = full_problem(name)
        T = TREES[name]
        model, margin = gbdt.train_problem(prob, n_trees=T)
        nodes = model.nodes()
        extra = {}
        if name == "C5":
            m_rle, y_rle = gbdt.train_problem(prob, n_trees=T, rle="on")
            extra["rle"] = (m_rle.nodes(), y_rle)
        res[name] = (prob, nodes, margin, pool.submit(_oracle_job, prob, nodes[:T], T), extra)
        if "rle" in extra:
            extra["rle_oracle"] = pool.submit(_oracle_job, prob, extra["rle"][0][:T], T)
    yield res
    timings = {}
    for name, (_, _, _, fut, _) in res.items():
        if fut.done() and fut.exception() is None:
            timings[name] = fut.result()[1]
    os.makedirs("gpurun_out", exist_ok=True)
    with open(os.path.join("gpurun_out", "oracle_fullsize.json"), "w") as f:
        json.dump({"nproc": os.cpu_count(), "cpu_model": _cpu_model(), "threads_concurrent": len(ORDER),
                   "configs": timings}, f, indent=1)
    pool.shutdown(wait=True, cancel_futures=True)


@pytest.mark.parametrize("name", ORDER)
def test_full_size_tree_for_tree(runs, name):
    prob, nodes, margin, fut, extra = runs[name]
    out, tim = fut.result()
    st = check(prob, nodes, margin, out)
    assert st["exact"] + st["near_tie"] > 0
    print(f"{name}: {TREES[name]} trees, {st}, oracle {tim['wall_s']:.1f} s")
    if "rle" in extra:                              # RLE on: its own follow-mode run
        rn, ry = extra["rle"]
        st2 = check(prob, rn, ry, extra["rle_oracle"].result()[0])
        print(f"{name} RLE: {st2}")
