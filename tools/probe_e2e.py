"""Probe (GPU box): wall time of repeated C3 gbdt_load_csr calls from pinned host buffers, to see
whether bench.py's e2e load cost is a first-call effect.  Not part of the product or the tests."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
from datagen import synth
from paper_conf_ipps_wenhkls18_b200 import gbdt

print("cpus", os.cpu_count(), "affinity", len(os.sched_getaffinity(0)))
prob = synth.make("C3")
pin = lambda a: torch.from_numpy(np.ascontiguousarray(a)).pin_memory().numpy()
hp, hi, hv, hl = pin(prob.indptr), pin(prob.indices), pin(prob.values), pin(prob.labels)
st = torch.cuda.current_stream()
for k in range(4):
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    ds = gbdt.load_csr(hp, hi, hv, hl, prob.m, stream=st.cuda_stream)
    torch.cuda.synchronize()
    t1 = time.perf_counter()
    print(f"load {k}: {t1 - t0:.3f} s", flush=True)
    del ds
    torch.cuda.synchronize()
