make -s -C oracle
for W in 0 1; do
GBDT_FUSEDW=$W GBDT_LIB=$PWD/paper_conf_ipps_wenhkls18_b200/libgbdt_dbg.so GBDT_FUSED=1 timeout 300 python -c "
import sys; sys.path.insert(0,'.')
import numpy as np
from datagen import synth
from paper_conf_ipps_wenhkls18_b200 import gbdt
p = synth.c3(n=60000, T=1)
m, y = gbdt.train_problem(p, max_depth=3)
np.save('gpurun_out/n3_w$W.npy', m.nodes())
" > gpurun_out/dbg_$W.log 2>&1
done
