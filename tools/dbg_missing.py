import sys
sys.path.insert(0, ".")
from datagen import synth
from paper_conf_ipps_wenhkls18_b200 import gbdt
p = synth.random_small(0, n=3000, m=5, nan_frac=0.3, n_distinct=50, loss="squared")
m, margin = gbdt.train_problem(p, n_trees=1)
print("ok", m.nodes()[0][:3])
