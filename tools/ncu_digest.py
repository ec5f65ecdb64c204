"""Digest of one ncu report: key metrics, stall reasons, dynamic opcode mix (usage: ncu_digest.py REP)."""
import csv, io, subprocess, sys
from collections import Counter
rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, units, vals = rows[0], rows[1], rows[2]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__occupancy_limit_registers",
        "launch__occupancy_limit_shared_mem", "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "lts__t_sector_hit_rate.pct", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed"]
for w in want:
    if w in h:
        i = h.index(w); print(f"{w:60s} {vals[i]:>20s} {units[i]}")
st = [(h[i], vals[i]) for i in range(len(h)) if h[i].startswith("smsp__pcsamp_warps_issue_stalled_") and not h[i].endswith("not_issued")]
tot = sum(float(v.replace(",", "") or 0) for _, v in st)
for k, v in sorted(st, key=lambda x: -float(x[1].replace(",", "") or 0))[:10]:
    print(f"  stall {k.replace('smsp__pcsamp_warps_issue_stalled_', ''):30s} {float(v.replace(',', ''))/max(tot,1)*100:5.1f}%")
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
R = list(csv.reader(io.StringIO(src)))
hh = R[1]; R = R[2:]
iS, iE = hh.index("Source"), hh.index("Instructions Executed")
c = Counter(); T = 0
for r in R:
    e = int(r[iE]) if r[iE].isdigit() else 0
    s = r[iS].strip()
    if s.startswith("@"): s = s.split(None, 1)[1] if " " in s else s
    op = s.split()[0].split(".")[0] if s else ""
    c[op] += e; T += e
print("dynamic warp instructions", T)
sys.stdout.flush(); print("  " + "  ".join(f"{k}:{v/T*100:.1f}%" for k, v in c.most_common(16)))
if len(sys.argv) > 2:
    with open(sys.argv[2], "w") as f:
        for i, r in enumerate(R):
            f.write(f"{i:5d} {r[iE]:>10s} {r[iS]}\n")
