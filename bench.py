#!/usr/bin/env python
"""Benchmark of the GPU-GBDT hot path on B200 (BASELINE.json metric: seconds per tree at depth 6;
split-find HBM GB/s vs peak).

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C3] [--impl ours|reference]

A step is one tree: one pass of the whole per-tree hot path (SmartGD gradients, then for every
level split finding, decision, node map and partition) over the resident synthetic dataset.
`value` = device seconds per tree of a K-tree gbdt_train (CUDA events on the library's stream,
max over ranks), after a W-tree warm-up training.  The dataset (2.5 GB of sorted lists for C3)
is larger than L2, so no flush is needed between steps.  `e2e` = the same metric through the C
ABI from pinned host buffers: gbdt_load_csr (H2D + layout build) + gbdt_train + margin D2H.
For N > 1 (torchrun) the attributes are sharded over the ranks (NCCL allgather of node bests +
bitmap allreduce per level) and the total work is fixed ("strong" scaling).

--impl reference times the CPU oracle (oracle/, single thread pinned to one core) on the FULL
rows of the same workload: presort once (excluded, reported), then the first K' trees (K' =
min(--steps, --ref-trees)); `steps` reports K' (the trees actually run).  cpu_baseline (our arm,
rank 0, N=1) is the same measurement with --cpu-trees trees.

roofline: SURVEY.md §8(d)'s algorithmic bytes per unit (one active entry at one level):
split find 24 B (logistic: val 4 + ins 4 + g/h 16; squared 16), partition 16 B (read 8 + write 8,
levels < d-1), node map 12 B per instance per level, gradient 40 B per instance per tree; the
level entries N_l come from the library (gbdt_get_level_entries).  `roofline` is the partition
phase (the phase furthest below its bound), per level: bytes / (phase ms per level); the split
phase and the whole tree are reported beside it.  The design's own streaming bytes and the ncu
DRAM bytes are side fields.
"""
import argparse
import json
import os
import statistics
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "seconds per tree (depth 6) at 1/2/4/8 B200; split-find HBM GB/s vs peak"
UNIT = "s/tree"
# SURVEY.md §8(d) algorithmic bytes (the unit: one active entry at one level)
def s8d_bytes(loss, rle):
    """(split B/entry, partition B/entry, nodemap B/instance/level, gradient B/instance/tree)."""
    gh = 8 if loss == "squared" else 16
    split = (4 + gh) if rle else (4 + 4 + gh)   # RLE: ins 4 + g/h (+ 8 B per run, not counted here)
    part = 8 if rle else 16                      # RLE: ins r/w (+ per-run bytes, not counted here)
    return split, part, 12, 40


# The design's own streaming bytes (g travels with the entries):
#   split find reads val 4 + g-list 8 per entry (+ h-list 8 when h is stored; RLE: no val)
#   partition reads val 4 + ins 4 + g 8 + side 1 per entry and writes val 4 + ins 4 + g 8 per kept entry
def design_bytes(rle):
    v = 0 if rle else 4
    return 8 + v, 13 + v, 12 + v


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C3")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--rle", default="off")
    ap.add_argument("--rle-split", default="direct", choices=["direct", "decompress"],
                    help="RLE node split: direct (P:250, Fig. 7) or the decompression ablation (P:248, Fig. 6)")
    ap.add_argument("--local-shards", type=int, default=int(os.environ.get("GBDT_LOCAL_SHARDS", "1")),
                    help="attribute shards inside this process (1, 2, 4 or 8; they pipeline on streams)")
    ap.add_argument("--dense", action="store_true",
                    help="dense representation, absent values filled with 0 (P:116, P:405-413, SURVEY §8(f4))")
    ap.add_argument("--comm", default="nccl", choices=["nccl", "host"],
                    help="host: gloo + host-staged callbacks (several ranks may share one GPU; testing only)")
    ap.add_argument("--depth", type=int, default=0, help="override the config's max_depth (sweeps, SURVEY §8(f2))")
    ap.add_argument("--smartgd", default="on", choices=["on", "off"],
                    help="off: SmartGD ablation, predictions recomputed by tree traversal (P:193-195, Fig. 9)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-trees", type=int, default=1, help="oracle trees (full rows) timed for cpu_baseline")
    ap.add_argument("--ref-trees", type=int, default=2, help="--impl reference: at most this many full-row trees")
    return ap.parse_args()


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return float(d["hbm_gbs"]), "measured"
    return 6650.0, "fallback"


def clock_sampler_start():
    try:
        return subprocess.Popen(
            ["nvidia-smi", "--query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
             "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap",
             "--format=csv,noheader,nounits", "-lms", "100"],
            stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
    except Exception:
        return None


def clock_sampler_stop(proc, dev=0):
    if proc is None:
        return None
    time.sleep(0.15)
    proc.terminate()
    try:
        out, _ = proc.communicate(timeout=5)
    except Exception:
        proc.kill()
        out = ""
    sm, smax, reasons = [], 0.0, set()
    names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
    for line in out.strip().splitlines():
        f = [x.strip() for x in line.split(",")]
        if len(f) < 9 or f[0] != str(dev):
            continue
        try:
            sm.append(float(f[1]))
            smax = max(smax, float(f[2]))
        except ValueError:
            continue
        for nm, v in zip(names, f[5:9]):
            if v.lower().startswith("active"):
                reasons.add(nm)
    if not sm:
        return None
    return {"sm_mhz": statistics.median(sm), "sm_max_mhz": smax, "reasons": sorted(reasons), "samples": len(sm)}


def host_info():
    model = ""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    return {"cpu_model": model, "nproc": os.cpu_count()}


def oracle_full_rows(prob, trees, depth):
    """The CPU oracle (single thread, pinned to one core) on the workload's full rows: presort once,
    then `trees` trees at `depth`.  Returns (seconds per tree, info)."""
    from oracle import oracle
    old = os.sched_getaffinity(0)
    core = max(old)
    os.sched_setaffinity(0, {core})  # this (calling) thread only
    try:
        t0 = time.perf_counter()
        oracle.train(prob, params=dict(n_trees=trees, max_depth=depth))
        wall = time.perf_counter() - t0
        presort, per_tree = oracle.last_timings()
    finally:
        os.sched_setaffinity(0, old)
    info = dict(trees=trees, presort_s=presort, tree_s=per_tree, wall_s=wall, core=core, **host_info())
    return sum(per_tree) / max(len(per_tree), 1), info


def arm_config(args, prob, P, d, world):
    """The `config` object of the JSON line; identical for both arms."""
    return {"workload": args.config, "n": prob.n, "m": prob.m, "nnz": prob.nnz, "loss": P["loss"],
            "max_depth": d, "trees_timed": args.steps, "lambda": P["lam"], "eta": P["eta"],
            "rle": args.rle, "rle_split": args.rle_split, "dense": args.dense, "smartgd": args.smartgd,
            "parallelism": f"attr-shard{world}",
            "l2": ("inputs larger than L2 (sorted lists %.2f GB)" % (prob.nnz * 8 / 1e9)) if prob.nnz * 8 > 126e6
                  else "inputs smaller than L2 (%.1f MB), not flushed between trees: latency-bound config"
                  % (prob.nnz * 8 / 1e6)}


def main():
    args = parse()
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    from datagen import synth

    if args.impl == "reference":
        if rank != 0:
            return
        prob = synth.make(args.config)
        P = prob.params
        d = args.depth or P["max_depth"]
        trees = max(1, min(args.steps, args.ref_trees))
        rate, info = oracle_full_rows(prob, trees, d)
        sample = (f"full rows ({prob.n} x {prob.m}, {prob.nnz} entries), first {trees} tree(s) at depth {d}, "
                  f"presort {info['presort_s']:.1f} s excluded; 1 thread pinned to core {info['core']} of "
                  f"{info['nproc']} ({info['cpu_model']})")
        line = {
            "impl": "reference", "metric": METRIC, "value": rate, "unit": UNIT, "n_gpus": args.gpus,
            "steps": trees, "steps_requested": args.steps, "warmup": 0, "ms_per_step": rate * 1e3,
            "higher_is_better": False, "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": arm_config(args, prob, P, d, world),
            "cpu_baseline": {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                             "tree_s": info["tree_s"], "presort_s": info["presort_s"]},
            "e2e": {"value": rate, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
        }
        print(json.dumps(line))
        return

    import torch
    host_comm = args.comm == "host"
    if host_comm:
        local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        if host_comm:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    from paper_conf_ipps_wenhkls18_b200 import gbdt

    def allmax(x):  # max over ranks of a host float
        t = torch.tensor([x], device="cpu" if host_comm else "cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    prob = synth.make(args.config)
    P = dict(prob.params)
    if args.depth:
        P["max_depth"] = args.depth
    d = P["max_depth"]
    comm = None
    if world > 1:
        comm = gbdt.comm_from_callbacks(local) if host_comm else gbdt.comm_from_torch(local)
    stream = torch.cuda.current_stream()
    ds = gbdt.load_csr(prob.indptr, prob.indices, prob.values, prob.labels, prob.m, rle=args.rle,
                       stream=stream.cuda_stream, comm=comm, keep_rows=args.smartgd == "off", dense=args.dense,
                       n_shards=args.local_shards)
    info = ds.info(0)
    m_local = info["attr_end"] - info["attr_begin"]
    tp = dict(max_depth=d, lam=P["lam"], gamma=P["gamma"], eta=P["eta"], base_margin=P["base_margin"],
              loss=P["loss"], smartgd=args.smartgd == "on", rle_split=args.rle_split)

    # warm-up (untimed)
    gbdt.train(ds, n_trees=max(args.warmup, 1), want_margin=False, **tp)
    torch.cuda.synchronize()
    if dist:
        dist.barrier()
    torch.cuda.synchronize()
    clk = clock_sampler_start()
    time.sleep(0.3)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record(stream)
    model, _ = gbdt.train(ds, n_trees=args.steps, want_margin=False, **tp)  # one CUDA graph per tree
    ev1.record(stream)
    torch.cuda.synchronize()
    clocks = clock_sampler_stop(clk, local)
    launches = gbdt.last_launch_count()
    ms = ev0.elapsed_time(ev1)
    if dist:
        ms = allmax(ms)
        dist.barrier()
    torch.cuda.synchronize()
    # the same K trees again with the per-phase / per-kernel event timers (launched eagerly; not
    # the headline number): roofline of the dominant kernels
    model, _ = gbdt.train(ds, n_trees=args.steps, want_margin=False, profile=True, **tp)
    torch.cuda.synchronize()
    tim = model.timings()
    nodes = model.nodes()
    ent = model.level_entries(d)                     # list entries per level, summed over the K trees
    peak, peak_kind = peaks()
    rle = args.rle != "off"
    sb, pb, nb, gb = s8d_bytes(P["loss"], rle)
    T = args.steps
    fused = os.environ.get("GBDT_FUSED", "0") not in ("", "0") and not rle
    # entries per level summed over the K trees: split find scans every level, the partition
    # levels 0 .. d-2; per-level (launch) averages divide by K
    split_bytes = float(ent.sum()) * sb
    part_bytes = float(ent[:-1].sum()) * pb
    tree_bytes = split_bytes + part_bytes + T * (nb * prob.n * d + gb * prob.n)
    traffic = None
    tp_path = os.path.join(ROOT, "profiles", f"ncu_phases_{args.config}.json")
    if os.path.exists(tp_path):
        with open(tp_path) as f:
            traffic = json.load(f)

    def phase(name, nbytes, ms_total, launches, note):
        per = nbytes / max(launches, 1)
        avg = ms_total / max(launches, 1)
        ach = (per / 1e9) / (avg / 1e3) if ms_total > 0 else None
        tr = traffic.get(name, {}).get("dram_bytes_per_launch") if traffic else None
        return {"achieved": ach, "frac": ach / peak if ach else None, "bytes_per_launch": per,
                "avg_launch_ms": avg, "launches": launches, "traffic": tr, "bytes_model": note}

    if fused:  # one pass per level: partition of level l + split find of level l+1 (fused.cu)
        part_ph = phase("partition", part_bytes + float(ent[1:].sum()) * sb, tim["partition"], T * (d - 1),
                        f"{pb} B/entry (partition, levels < d-1) + {sb} B/entry (split find of levels >= 1)")
        split_ph = phase("split_find", float(ent[0]) * sb, tim["split_find"], T, f"{sb} B/entry, root level")
    else:
        part_ph = phase("partition", part_bytes, tim["partition"], T * (d - 1), f"{pb} B/entry, levels < d-1")
        split_ph = phase("split_find", split_bytes, tim["split_find"], T * d, f"{sb} B/entry, every level")
    tree_ph = phase("tree", tree_bytes, ms, T,
                    f"§8(d): {sb} B/entry/level split + {pb} B/entry/level partition + {nb} B/instance/level "
                    f"node map + {gb} B/instance gradient")
    # the design's own streaming bytes (g travels with the entries) as a side field
    d_split, d_sread, d_swrite = design_bytes(rle)
    design = {"split_find_B_per_entry": d_split, "partition_B_per_entry": f"{d_sread} read + {d_swrite} per kept entry",
              "split_find_GBps": (float(ent.sum()) * d_split / 1e9) / (tim["split_find"] / 1e3) if tim["split_find"] else None,
              "partition_GBps": ((float(ent[:-1].sum()) * d_sread + float(ent[1:].sum()) * d_swrite) / 1e9) /
                                (tim["partition"] / 1e3) if tim["partition"] and not fused else None}
    # e2e through the C ABI from pinned host buffers
    e2e = None
    if not args.no_e2e:
        # the device-resident dataset goes back to the library's stream-ordered pool first, as in
        # a process that trains dataset after dataset: the e2e load then reuses that memory instead
        # of growing the pool by another copy of the layout while the first one is still held
        # (which cost 0.3-1.1 s per 40 trees on C3, varying from box to box)
        del ds
        import gc
        gc.collect()
        torch.cuda.synchronize()
        pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory().numpy()
        hp, hi, hv, hl = pin(prob.indptr), pin(prob.indices), pin(prob.values), pin(prob.labels)
        if dist:
            dist.barrier()
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        ds2 = gbdt.load_csr(hp, hi, hv, hl, prob.m, rle=args.rle, stream=stream.cuda_stream, comm=comm,
                            keep_rows=args.smartgd == "off", dense=args.dense, n_shards=args.local_shards)
        model2, margin2 = gbdt.train(ds2, n_trees=args.steps, want_margin=True, **tp)
        torch.cuda.synchronize()
        te = time.perf_counter() - t0
        if dist:
            te = allmax(te)
        h2d = hp.nbytes + hi.nbytes + hv.nbytes + hl.nbytes
        d2h = margin2.nbytes + nodes.nbytes
        e2e = {"value": te / args.steps, "unit": UNIT, "h2d_bytes_per_step": int(h2d / args.steps),
               "d2h_bytes_per_step": int(d2h / args.steps),
               "note": "one gbdt_load_csr (H2D + layout sort) + K-tree gbdt_train + margin D2H, amortised per tree; "
                       "library memory pool warm (the device-timed run's dataset was freed into it first)"}
        del ds2, model2

    # gbdt_predict on the training rows with the K trees: wall clock through the
    # C ABI, the CSR's H2D copy included; must reproduce the training margin
    pred = None
    if rank == 0 and world == 1 and not args.no_e2e:
        hp_, hi_, hv_ = [torch.from_numpy(np.ascontiguousarray(a)).pin_memory().numpy()
                         for a in (prob.indptr, prob.indices, prob.values)]
        model.predict(hp_, hi_, hv_, prob.m)  # warm-up
        t0 = time.perf_counter()
        model.predict(hp_, hi_, hv_, prob.m)
        tp_s = time.perf_counter() - t0
        pred = {"rows_per_s": prob.n / tp_s, "s": tp_s, "trees": args.steps,
                "note": "gbdt_predict on the training rows, CSR H2D + D2H included"}

    cpu = None
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        rate, cinfo = oracle_full_rows(prob, max(1, args.cpu_trees), d)
        cpu = {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"full rows ({prob.n} x {prob.m}, {prob.nnz} entries), first {cinfo['trees']} tree(s) at "
                         f"depth {d}, presort {cinfo['presort_s']:.1f} s excluded; 1 thread pinned to core "
                         f"{cinfo['core']} of {cinfo['nproc']} ({cinfo['cpu_model']})",
               "tree_s": cinfo["tree_s"], "presort_s": cinfo["presort_s"]}

    if rank == 0:
        value = ms / 1e3 / args.steps
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": False,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": arm_config(args, prob, P, d, world),
            "roofline": {"bound": "hbm", "achieved": part_ph["achieved"], "peak": peak, "unit": "GB/s",
                         "frac": part_ph["frac"], "traffic": part_ph["traffic"],
                         "kernel": "partition phase (per level)" + (" = fused partition + next-level split find" if fused else
                                   ": k_part_count* + count scans + plan + k_part_scatter"),
                         "peak_kind": peak_kind, "bytes_per_launch": part_ph["bytes_per_launch"],
                         "launches": part_ph["launches"], "avg_launch_ms": part_ph["avg_launch_ms"],
                         "bytes_model": part_ph["bytes_model"],
                         "phases": {"split_find": split_ph, "partition": part_ph, "tree": tree_ph},
                         "design_bytes": design, "level_entries": [int(x) for x in ent]},
            "phases_ms_per_tree": {k: v / args.steps for k, v in tim.items()},
            "phases_note": "profiled re-run of the same K trees (event timers, eager launches)",
            "cpu_baseline": cpu,
            "e2e": e2e,
            "gpu_launches": launches,
            "predict": pred,
            "clocks": clocks,
            "context": {"paper_gpu_gbdt_titanx_higgs10M_mse_s_per_tree": 5.50,
                        "paper_xgbst40_higgs10M_mse_s_per_tree": 9.66, "source": "PAPER.md P:478-487 /40"},
        }
        print(json.dumps(line))
    if dist:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
