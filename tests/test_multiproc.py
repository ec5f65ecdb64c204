"""Host logic of the attribute-sharded multi-GPU path, on CPU.

* shard_ranges: the P-way attribute partition every rank computes independently must be a
  contiguous cover of [0, m), identical on every rank, and balanced by entries.
* the NCCL unique-id bootstrap over torch.distributed (rank 0 creates, everyone receives the
  same 128 bytes) -- world_size 2, gloo.
* the host-staged collectives used by gbdt_comm_init_callbacks (allgather in rank order,
  uint8 sum-allreduce) -- world_size 2, gloo.
"""
import ctypes as C
import os
import socket

import numpy as np
import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_ipps_wenhkls18_b200 import gbdt


def _zipf_counts(seed, m):
    rng = np.random.default_rng(seed)
    return np.floor(rng.pareto(1.1, m) * 5).astype(np.int64)


@pytest.mark.parametrize("P", [1, 2, 4, 8])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_shard_ranges_cover_and_balance(P, seed):
    m = 50 + 97 * seed
    cc = _zipf_counts(seed, m)
    b = gbdt.shard_ranges(cc, P)
    assert b[0] == 0 and b[-1] == m and np.all(np.diff(b) >= 0)
    pre = np.concatenate([[0], np.cumsum(cc)])
    tot = pre[-1]
    # greedy prefix targets: boundary i is the first attribute whose prefix reaches i/P of the
    # entries, so every shard holds at most tot/P + (its largest column) entries
    for i in range(1, P):
        assert pre[b[i]] >= tot * i / P or b[i] == m
        assert b[i] == b[i - 1] or pre[b[i] - 1] < tot * i / P
    for i in range(P):
        load = pre[b[i + 1]] - pre[b[i]]
        biggest = cc[b[i]:b[i + 1]].max() if b[i + 1] > b[i] else 0
        assert load <= tot / P + biggest + 1e-9


def test_shard_ranges_rejects_bad_world():
    with pytest.raises(gbdt.GbdtError):
        gbdt.shard_ranges(np.ones(4, np.int64), 3)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        # 1. identical shard ranges on every rank
        cc = _zipf_counts(7, 333)
        b = gbdt.shard_ranges(cc, world)
        import torch
        allb = [torch.zeros(world + 1, dtype=torch.int32) for _ in range(world)]
        dist.all_gather(allb, torch.from_numpy(b))
        ok_ranges = all(np.array_equal(x.numpy(), b) for x in allb)
        # 2. NCCL id bootstrap: rank 0's id reaches every rank unchanged
        uid = gbdt.comm_unique_id() if rank == 0 else bytes(128)
        t = torch.tensor(list(uid), dtype=torch.uint8)
        dist.broadcast(t, 0)
        got = bytes(t.tolist())
        ids = [torch.zeros(128, dtype=torch.uint8) for _ in range(world)]
        dist.all_gather(ids, t)
        ok_id = all(bytes(x.tolist()) == got for x in ids) and got != bytes(128)
        # 3. host-staged collectives (what the library calls through gbdt_comm_init_callbacks)
        ag, ar = gbdt.torch_collectives()
        send = (C.c_uint8 * 5)(*[rank * 10 + i for i in range(5)])
        recv = (C.c_uint8 * (5 * world))()
        rc1 = ag(C.addressof(send), C.addressof(recv), 5, None)
        ok_ag = rc1 == 0 and list(recv) == [r * 10 + i for r in range(world) for i in range(5)]
        buf = (C.c_uint8 * 6)(*[(1 if (i % world) == rank else 0) for i in range(6)])
        rc2 = ar(C.addressof(buf), 6, None)
        ok_ar = rc2 == 0 and list(buf) == [1] * 6
        out[rank] = int(ok_ranges) + 2 * int(ok_id) + 4 * int(ok_ag) + 8 * int(ok_ar)
    finally:
        dist.destroy_process_group()


def test_gloo_two_ranks_host_logic():
    world = 2
    ctx = mp.get_context("spawn")
    out = ctx.Array("i", [0] * world)
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, out)) for r in range(world)]
    for p in procs:
        p.start()
    for p in procs:
        p.join(120)
        assert p.exitcode == 0
    assert list(out) == [15] * world, list(out)
