"""B200-native exact-greedy GBDT hot path (GPU-GBDT, Wen et al., IPDPS 2018).

The product is the C-ABI library ``libgbdt.so`` (include/gbdt.h) built from ``csrc/`` for
sm_100a; :mod:`paper_conf_ipps_wenhkls18_b200.gbdt` is its ctypes binding.
"""
from . import gbdt  # noqa: F401
from .gbdt import load_csr, predict, train  # noqa: F401
