"""Turn the ncu outputs of tools/profile_round.sh into the committed profiles/ summaries.

usage: python tools/ncu_summary.py CFG ROUND   (reads gpurun_out/, writes profiles/)
  profiles/<ROUND>_launches_<CFG>.csv            the raw launch list (one tree)
  profiles/<ROUND>_launches_<CFG>_tree.txt       per-kernel totals of the last tree
  profiles/<ROUND>_<kernel>_<CFG>_ncu_full.txt   key metrics of one --set full capture
  profiles/ncu_<k_split|k_scatter>_<CFG>.json    DRAM bytes per launch (bench.py 'traffic')
"""
import collections
import csv
import json
import os
import shutil
import subprocess
import sys

cfg, rnd = sys.argv[1], sys.argv[2]
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
go, pr = os.path.join(root, "gpurun_out"), os.path.join(root, "profiles")
ll = os.path.join(go, f"launches_{cfg}.csv")
shutil.copy(ll, os.path.join(pr, f"{rnd}_launches_{cfg}.csv"))
tree = subprocess.run([sys.executable, os.path.join(root, "tools", "launch_summary.py"), ll],
                      capture_output=True, text=True).stdout
open(os.path.join(pr, f"{rnd}_launches_{cfg}_tree.txt"), "w").write(tree)

# per-launch DRAM bytes of the last tree
lines = open(ll).read().splitlines()
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
grads = [i for i in ids if "k_grad" in d[i]["name"]]
last = [i for i in ids if i >= (grads[-1] if grads else 0)]
groups = {"k_split": ("k_sf_fast", "k_sf_gen"), "k_scatter": ("k_part_scatter", "k_run_count", "k_run_scatter")}
for gname, pref in groups.items():
    # launches grouped per level: k_split = one k_sf_fast (+ its k_sf_gen); k_scatter = one k_part_scatter
    lead = pref[0]
    n_lead = sum(1 for i in last if d[i]["name"].split("(")[0].split("::")[-1].startswith(lead))
    byts = sum(d[i].get("dram__bytes_read.sum", 0) + d[i].get("dram__bytes_write.sum", 0) for i in last
               if any(d[i]["name"].split("(")[0].split("::")[-1].startswith(p) for p in pref))
    ms = sum(d[i].get("gpu__time_duration.sum", 0) for i in last
             if any(d[i]["name"].split("(")[0].split("::")[-1].startswith(p) for p in pref)) / 1e6
    if n_lead:
        json.dump({"source": f"ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                             f"--clock-control none (profiles/{rnd}_launches_{cfg}.csv), last tree of "
                             f"bench.py --config {cfg} --steps 1",
                   "kernels": list(pref), "launches": n_lead, "dram_bytes_per_launch": byts / n_lead,
                   "ncu_ms_per_launch": ms / n_lead},
                  open(os.path.join(pr, f"ncu_{gname}_{cfg}.json"), "w"), indent=1)

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__inst_executed.sum", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "launch__grid_size",
        "lts__t_sector_hit_rate.pct", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active"]
for k in ("k_sf_fast", "k_part_scatter", "k_chunk_agg", "k_part_count"):
    rep = os.path.join(go, f"full_{k}_{cfg}.ncu-rep")
    if not os.path.exists(rep):
        continue
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(out.splitlines()))
    hh, vv = r[0], r[2]
    lines = [f"ncu --set full --clock-control none -k regex:{k} -s 2 -c 1  (bench.py --config {cfg})",
             f"kernel: {vv[hh.index('Kernel Name')]}"]
    for key in KEYS:
        if key in hh:
            lines.append(f"{key:60s} {vv[hh.index(key)]}")
    stalls = [(x, float(vv[i])) for i, x in enumerate(hh)
              if x.startswith("smsp__pcsamp_warps_issue_stalled") and not x.endswith("not_issued") and vv[i]]
    tot = sum(v for _, v in stalls) or 1
    lines.append("stall samples (share):")
    for x, v in sorted(stalls, key=lambda t: -t[1])[:8]:
        lines.append(f"  {x.replace('smsp__pcsamp_warps_issue_stalled_', ''):30s} {100 * v / tot:5.1f}%")
    open(os.path.join(pr, f"{rnd}_{k}_{cfg}_ncu_full.txt"), "w").write("\n".join(lines) + "\n")
print(tree)
