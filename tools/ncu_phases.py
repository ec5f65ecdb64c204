"""Per-phase DRAM bytes of one tree from an ncu launch list (gpu__time_duration.sum,
dram__bytes_read.sum, dram__bytes_write.sum per launch) -> profiles/ncu_phases_<CFG>.json, the
`traffic` of bench.py's roofline phases.  Only the last tree of the list (after the last k_grad).

usage: python tools/ncu_phases.py LAUNCHES.csv CFG DEPTH [OUT.json]
"""
import collections
import csv
import json
import os
import sys


def short(name):
    return name.split("(")[0].split("::")[-1]


def phase_of(name):
    n = short(name)
    if n.startswith(("k_chunk_agg", "k_desc", "k_sf_", "k_seg_totals", "k_short_split", "k_run_root", "k_run_agg",
                     "k_run_init", "k_run_split")) or n.startswith("k_scan") and "<1>" in n:
        return "split_find"
    if n.startswith(("k_part_", "k_plan_", "k_chunk_attr", "k_run_", "k_tile_agg", "k_tscan", "k_fused")) or \
            n.startswith("k_scan") and "<0>" in n:
        return "partition"
    if n.startswith(("k_mark", "k_nodemap")):
        return "nodemap"
    if n.startswith(("k_pick", "k_decide", "k_level_begin")):
        return "decide"
    if n.startswith(("k_grad", "k_tree_begin", "k_apply", "k_tree_end")):
        return "grad"
    return "other"


def main():
    path, cfg, depth = sys.argv[1], sys.argv[2], int(sys.argv[3])
    out = sys.argv[4] if len(sys.argv) > 4 else os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                                           "profiles", f"ncu_phases_{cfg}.json")
    lines = open(path).read().splitlines()
    start = next(i for i, l in enumerate(lines) if l.startswith('"ID"'))
    rows = list(csv.reader(lines[start:]))
    h = rows[0]
    iK, iM, iV, iID = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    d = collections.defaultdict(dict)
    for r in rows[1:]:
        if len(r) == len(h):
            d[int(r[iID])][r[iM]] = float(r[iV].replace(",", ""))
            d[int(r[iID])]["name"] = r[iK]
    ids = sorted(d)
    grads = [i for i in ids if short(d[i]["name"]).startswith("k_grad")]
    last = [i for i in ids if i >= grads[-1]] if grads else ids
    agg = collections.defaultdict(lambda: [0.0, 0.0, 0])
    for i in last:
        ph = phase_of(d[i]["name"])
        a = agg[ph]
        a[0] += d[i].get("dram__bytes_read.sum", 0) + d[i].get("dram__bytes_write.sum", 0)
        a[1] += d[i].get("gpu__time_duration.sum", 0) / 1e6  # ns -> ms
        a[2] += 1
    levels = {"split_find": depth, "partition": depth - 1, "nodemap": depth, "decide": depth, "grad": 1, "other": 1}
    res = {"source": f"ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                     f"--clock-control none, last tree of {os.path.basename(path)} (cold-cache, serialised)"}
    for ph, (b, ms, n) in agg.items():
        res[ph] = {"dram_bytes_per_launch": b / levels.get(ph, 1), "ncu_ms_per_launch": ms / levels.get(ph, 1),
                   "kernel_launches": n, "launches_per_tree": levels.get(ph, 1)}
    tree_b = sum(v[0] for v in agg.values())
    res["tree"] = {"dram_bytes_per_launch": tree_b, "ncu_ms_per_launch": sum(v[1] for v in agg.values())}
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
