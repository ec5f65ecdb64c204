import json, sys, glob
for f in sorted(glob.glob("gpurun_out/bench_*.log")):
    for l in open(f):
        if l.startswith("{"):
            d = json.loads(l); k = d["roofline"]["kernels"]; ph = d["phases_ms_per_tree"]
            print(f"{d['config']['workload']:4s} {d['value']*1e3:8.3f} ms/tree | split {k['k_split']['avg_launch_ms']:.3f} ms {k['k_split']['frac']:.3f} | "
                  f"scatter {k['k_scatter']['avg_launch_ms']:.3f} ms {k['k_scatter']['frac']:.3f} | " +
                  " ".join(f"{x}={ph[x]:.2f}" for x in ["grad","k_chunk_agg","k_split","k_count","k_scatter","decide","nodemap"]))
