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

--impl reference times the CPU oracle (oracle/, single thread) on a bounded row sample of the
same workload and scales it to the full workload's entries (the paper's cost model is linear in
the number of entries per level).
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
# Algorithmic bytes of the two streaming kernels:
#   k_split   (k_sf_fast + k_sf_gen) per entry of the level: value f32 4 + g-list fp64 8
#             (+ h-list 8 when h is not a function of g; RLE: the runs replace the 4 value bytes)
#   k_scatter per entry of the level: val 4 + ins 4 + g 8 + side 1 read; per kept entry (the
#             next level's entries): val 4 + ins 4 + g 8 written
#   with RLE the 4 value bytes are not streamed (values come from the runs, a few bytes per run)
def byte_model(rle):
    v = 0 if rle else 4
    return 8 + v, 13 + v, 12 + v   # split per entry; scatter read per entry, write per kept entry


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=40)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C3")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--rle", default="off")
    ap.add_argument("--comm", default="nccl", choices=["nccl", "host"],
                    help="host: gloo + host-staged callbacks (several ranks may share one GPU; testing only)")
    ap.add_argument("--depth", type=int, default=0, help="override the config's max_depth (sweeps, SURVEY §8(f2))")
    ap.add_argument("--smartgd", default="on", choices=["on", "off"],
                    help="off: SmartGD ablation, predictions recomputed by tree traversal (P:193-195, Fig. 9)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-seconds", type=float, default=15.0, help="target oracle CPU time for cpu_baseline")
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


def oracle_sample_rate(prob, target_s, trees=2):
    """Oracle seconds per tree on the full workload, estimated from a bounded row sample."""
    from datagen import synth
    from oracle import oracle
    n_s = min(prob.n, 20000)
    while True:
        sub = _rows(prob, n_s)
        t0 = time.perf_counter()
        oracle.presort(sub.indptr, sub.indices, sub.values, sub.n, sub.m)
        t1 = time.perf_counter()
        oracle.train(sub, params=dict(n_trees=trees))
        t2 = time.perf_counter()
        per_tree = max((t2 - t1) - (t1 - t0), 1e-9) / trees
        if t2 - t0 > target_s / 4 or n_s >= prob.n:
            break
        n_s = min(prob.n, int(n_s * min(8.0, max(2.0, (target_s / 4) / max(t2 - t0, 1e-3)))))
    scale = prob.nnz / sub.nnz
    return per_tree * scale, dict(n_rows=n_s, entries=sub.nnz, trees=trees, per_tree_s=per_tree,
                                  scale=scale, presort_s=t1 - t0), synth


def _rows(prob, n_s):
    from datagen import synth
    if n_s >= prob.n:
        return prob
    e = int(prob.indptr[n_s])
    return synth.Problem(prob.name + f"[:{n_s}]", n_s, prob.m, prob.indptr[:n_s + 1].copy(),
                         prob.indices[:e], prob.values[:e], prob.labels[:n_s], prob.params)


def arm_config(args, prob, P, d, world):
    """The `config` object of the JSON line; identical for both arms."""
    return {"workload": args.config, "n": prob.n, "m": prob.m, "nnz": prob.nnz, "loss": P["loss"],
            "max_depth": d, "trees_timed": args.steps, "lambda": P["lam"], "eta": P["eta"],
            "rle": args.rle, "smartgd": args.smartgd, "parallelism": f"attr-shard{world}",
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
        from oracle import oracle
        # warm-up: W trees on a small sample (untimed), then the bounded timed sample
        sub = _rows(prob, min(prob.n, 2000))
        oracle.train(sub, params=dict(n_trees=max(1, min(args.warmup, 3))))
        rate, info, _ = oracle_sample_rate(prob, args.cpu_seconds * 2, trees=min(args.steps, 3))
        line = {
            "impl": "reference", "metric": METRIC, "value": rate, "unit": UNIT, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": rate * 1e3, "higher_is_better": False,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": arm_config(args, prob, P, args.depth or P["max_depth"], world),
            "cpu_baseline": {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle",
                             "sample": f"first {info['n_rows']} rows ({info['entries']} entries), "
                                       f"{info['trees']} trees, presort excluded, scaled x{info['scale']:.1f} by entries"},
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
                       stream=stream.cuda_stream, comm=comm, keep_rows=args.smartgd == "off")
    info = ds.info(0)
    m_local = info["attr_end"] - info["attr_begin"]
    tp = dict(max_depth=d, lam=P["lam"], gamma=P["gamma"], eta=P["eta"], base_margin=P["base_margin"],
              loss=P["loss"], smartgd=args.smartgd == "on")

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
    b_split, b_sread, b_swrite = byte_model(args.rle != "off")
    kern = {
        "k_split": dict(bytes=float(ent.sum()) * b_split, launches=args.steps * d,
                        ms=tim["k_split"], bytes_per_entry=b_split),
        "k_scatter": dict(bytes=float(ent[:-1].sum()) * b_sread + float(ent[1:].sum()) * b_swrite,
                          launches=args.steps * (d - 1), ms=tim["k_scatter"],
                          bytes_per_entry=f"{b_sread} read + {b_swrite} per kept entry"),
    }
    for kname, kv in kern.items():
        kv["avg_launch_ms"] = kv["ms"] / kv["launches"]
        kv["achieved"] = (kv["bytes"] / kv["launches"] / 1e9) / (kv["avg_launch_ms"] / 1e3) if kv["ms"] > 0 else None
        kv["frac"] = kv["achieved"] / peak if kv["achieved"] else None
        kv["traffic"] = None
        tp_path = os.path.join(ROOT, "profiles", f"ncu_{kname}_{args.config}.json")
        if os.path.exists(tp_path):
            with open(tp_path) as f:
                kv["traffic"] = json.load(f).get("dram_bytes_per_launch")
    dom = max(kern, key=lambda k: kern[k]["ms"])

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
                            keep_rows=args.smartgd == "off")
        model2, margin2 = gbdt.train(ds2, n_trees=args.steps, want_margin=True, **tp)
        torch.cuda.synchronize()
        te = time.perf_counter() - t0
        if dist:
            te = allmax(te)
        h2d = hp.nbytes + hi.nbytes + hv.nbytes + hl.nbytes
        d2h = margin2.nbytes + nodes.nbytes
        e2e = {"value": te / args.steps, "unit": UNIT, "h2d_bytes_per_step": int(h2d / args.steps),
               "d2h_bytes_per_step": int(d2h / args.steps),
               "note": "one gbdt_load_csr (H2D + layout sort) + K-tree gbdt_train + margin D2H, amortised per tree"}
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
        rate, cinfo, _ = oracle_sample_rate(prob, args.cpu_seconds)
        cpu = {"value": rate, "unit": UNIT, "cores": 1, "kind": "oracle",
               "sample": f"first {cinfo['n_rows']} rows ({cinfo['entries']} entries), {cinfo['trees']} trees, "
                         f"presort excluded, scaled x{cinfo['scale']:.1f} by entries"}

    if rank == 0:
        value = ms / 1e3 / args.steps
        line = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": ms / args.steps, "higher_is_better": False,
            "scaling": "strong", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": arm_config(args, prob, P, d, world),
            "roofline": {"bound": "hbm", "achieved": kern[dom]["achieved"], "peak": peak, "unit": "GB/s",
                         "frac": kern[dom]["frac"], "traffic": kern[dom]["traffic"], "kernel": dom,
                         "peak_kind": peak_kind, "bytes_per_launch": kern[dom]["bytes"] / kern[dom]["launches"],
                         "launches": kern[dom]["launches"], "avg_launch_ms": kern[dom]["avg_launch_ms"],
                         "kernels": {k: {kk: vv for kk, vv in v.items() if kk != "bytes"} for k, v in kern.items()}},
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
