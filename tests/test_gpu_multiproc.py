"""The attribute-sharded path across PROCESSES on one GPU: world_size 2 and 4
ranks share cuda:0 and exchange through gbdt_comm_init_callbacks over torch.distributed/gloo
(NCCL refuses two ranks on one device).  Every rank builds only its attribute shard, finds its
local bests, and the allgather + deterministic argmax + bitmap allreduce must reproduce the
single-process trees and margins bit for bit (-m gpu)."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _problem(name):
    from datagen import synth
    if name == "c2":
        return synth.c2(n=15000, T=3)
    return synth.c4(seed=11, n=1500, m=2000, density=0.01, T=2)


def _worker(rank, world, port, name, path):
    import torch.distributed as dist
    from paper_conf_ipps_wenhkls18_b200 import gbdt
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        p = _problem(name)
        comm = gbdt.comm_from_callbacks(device=0)
        P = dict(p.params)
        ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m, comm=comm, device=0)
        model, margin = gbdt.train(ds, **P)
        if rank == 0:
            np.save(path + ".nodes.npy", model.nodes().view(np.uint8))
            np.save(path + ".margin.npy", margin)
        dist.barrier()
        del model, ds
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name,world", [("c2", 2), ("c4", 2), ("c2", 4)])
def test_ranks_reproduce_single_process(tmp_path, name, world):
    from paper_conf_ipps_wenhkls18_b200 import gbdt
    p = _problem(name)
    ref_model, ref_margin = gbdt.train_problem(p)
    path = str(tmp_path / "r0")
    ctx = mp.get_context("spawn")
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, name, path)) for r in range(world)]
    for q in procs:
        q.start()
    for q in procs:
        q.join(600)
        assert q.exitcode == 0
    nodes = np.load(path + ".nodes.npy")
    margin = np.load(path + ".margin.npy")
    assert np.array_equal(nodes, ref_model.nodes().view(np.uint8))
    assert np.array_equal(margin, ref_margin)


@pytest.mark.parametrize("graph", ["0", "1"])
def test_nccl_world_of_one_runs_the_collectives(graph, monkeypatch):
    """The NCCL path on one GPU: a world of one rank makes the same ncclAllGather / ncclAllReduce
    calls per level (eager, or captured into the per-tree CUDA graph) and must reproduce the
    communicator-free model bit for bit."""
    import numpy as np
    from datagen import synth
    from paper_conf_ipps_wenhkls18_b200 import gbdt
    monkeypatch.setenv("GBDT_GRAPH", graph)
    p = synth.c1(n=3000)
    m0, y0 = gbdt.train_problem(p)
    comm = gbdt.comm_init(0, 1, gbdt.comm_unique_id(), 0)
    ds = gbdt.load_csr(p.indptr, p.indices, p.values, p.labels, p.m, comm=comm)
    P = dict(p.params)
    m1, y1 = gbdt.train(ds, **P)
    assert m0.nodes().tobytes() == m1.nodes().tobytes()
    assert np.array_equal(y0, y1)
    del ds
