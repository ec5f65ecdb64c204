"""One line per bench log: config, s/tree, roofline frac, per-phase ms/tree."""
import glob, json, sys
for f in sorted(sys.argv[1:] or glob.glob("gpurun_out/bench*.log")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "unparsed", e); continue
    ph = {k: round(v, 2) for k, v in d.get("phases_ms_per_tree", {}).items() if v}
    print(f.split("/")[-1], d["config"].get("workload"), round(d["value"] * 1e3, 3), "ms/tree",
          "frac", round(d.get("roofline", {}).get("frac") or 0, 3), ph)
