"""Executed instructions / stall samples per CUDA source line of one kernel (ncu SASS source page
CSV + the local cubin's line table).  usage: sass_lines.py OBJ KERNEL_REGEX NCU_SRC_CSV [N]"""
import collections, csv, os, re, subprocess, sys, tempfile
obj, kre, src_csv = sys.argv[1:4]
N = int(sys.argv[4]) if len(sys.argv) > 4 else 40
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=d, capture_output=True)
cub = [f for f in os.listdir(d) if f.endswith(".cubin")][0]
sass = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(d, cub)], capture_output=True, text=True).stdout
cur = None; m = {}; on = False
for l in sass.splitlines():
    if l.startswith(".text.") or "\t.section\t.text." in l:
        on = re.search(kre, l) is not None
    if not on:
        continue
    mm = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if mm:
        cur = (os.path.basename(mm.group(1)), int(mm.group(2))); continue
    mo = re.search(r'/\*([0-9a-f]{4,})\*/', l)
    if mo and cur:
        m.setdefault(int(mo.group(1), 16), cur)
rows = list(csv.reader(open(src_csv)))
h = rows[1]; data = [r for r in rows[2:] if len(r) > 10]
iA = h.index('Address'); iE = h.index('Instructions Executed'); iW = h.index('Warp Stall Sampling (All Samples)')
a0 = int(data[0][iA], 16)
agg = collections.Counter(); st = collections.Counter()
for r in data:
    k = m.get(int(r[iA], 16) - a0, ('?', 0))
    agg[k] += float(r[iE] or 0); st[k] += float(r[iW] or 0)
tot = sum(agg.values()) or 1; tst = sum(st.values()) or 1
srcs = {}
def line(f, n):
    for root in ("paper_conf_ipps_wenhkls18_b200/csrc",):
        p = os.path.join(root, f)
        if os.path.exists(p):
            srcs.setdefault(p, open(p).read().splitlines())
            return srcs[p][n - 1].strip()[:80]
    return ""
print(f"total {tot/1e6:.0f}M instr")
for k, v in agg.most_common(N):
    print(f"{k[0]:12s}{k[1]:5d} {v/1e6:7.1f}M {100*v/tot:4.1f}% st {100*st[k]/tst:4.1f}%  {line(*k)}")
