make -s -j8 -C paper_conf_ipps_wenhkls18_b200/csrc >/dev/null 2>&1; make -s -C oracle
for W in 0 1; do
GBDT_FUSEDW=$W GBDT_FUSED=1 timeout 600 compute-sanitizer --tool memcheck --print-limit 3 python -c "
import sys; sys.path.insert(0,'.'); sys.path.insert(0,'tests')
from datagen import synth
from paper_conf_ipps_wenhkls18_b200 import gbdt
p = synth.c3(n=60000, T=1)
m, y = gbdt.train_problem(p)
import numpy as np
np.save('gpurun_out/nodes_w$W.npy', m.nodes())
print('ok')
" > gpurun_out/san_w$W.log 2>&1
done
