import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from datagen import synth
from oracle import oracle
from paper_conf_ipps_wenhkls18_b200 import gbdt
p = synth.table1(loss="squared", d=2, T=2, lam=1.0, eta=1.0)
model, margin = gbdt.train_problem(p)
nodes = model.nodes()
on, om, st = oracle.train(p, follow=nodes)
o2, om2, _ = oracle.train(p)
np.set_printoptions(linewidth=200)
for t in range(2):
    for k in range(7):
        a = nodes[t, k]; b = o2[t, k]
        if a["heap_id"] >= 0 or b["heap_id"] >= 0:
            print(t, k, "GPU", a["is_leaf"], a["attr"], a["split_value"], a["default_left"], a["gain"], a["G"], a["H"], a["count"], a["weight"])
            print(t, k, "ORC", b["is_leaf"], b["attr"], b["split_value"], b["default_left"], b["gain"], b["G"], b["H"], b["count"], b["weight"], on[t,k]["follow_status"])
print(margin, om2, st)
