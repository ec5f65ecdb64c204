"""C-ABI boundary checks that need no GPU: the library builds, loads, exports every symbol that
include/gbdt.h declares, validates its inputs, and fails loudly (no CPU fallback) without a GPU."""
import ctypes as C
import os
import re

import numpy as np
import pytest

from paper_conf_ipps_wenhkls18_b200 import gbdt

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "gbdt.h")


def _declared():
    src = open(HEADER).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(gbdt_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_three_entry_points():
    names = _declared()
    for n in ("gbdt_load_csr", "gbdt_train", "gbdt_predict"):
        assert n in names


def test_library_exports_every_declared_symbol():
    L = gbdt.lib()
    missing = [n for n in _declared() if not hasattr(L, n)]
    assert not missing, missing


def test_nodes_dtype_matches_header_layout():
    assert gbdt.NODE_DTYPE.itemsize == 64
    assert gbdt.NODE_DTYPE.fields["gain"][1] == 24 and gbdt.NODE_DTYPE.fields["count"][1] == 56


def _load(indptr, indices, values, labels, n_cols):
    L = gbdt.lib()
    h = C.c_void_p()
    o = gbdt._LoadOpts(0, 0.0, 1, -1, None, None)
    a = [np.ascontiguousarray(x) for x in (indptr, indices, values, labels)]
    st = L.gbdt_load_csr(a[0].size - 1, n_cols, *[x.ctypes.data_as(C.c_void_p) for x in a], C.byref(o), C.byref(h))
    return st, h.value, L.gbdt_last_error().decode()


@pytest.mark.parametrize("case,expect", [
    (dict(indptr=[1, 2], indices=[0], values=[1.0], labels=[0.0], n_cols=1), "indptr[0]"),
    (dict(indptr=[0, 2, 1], indices=[0, 1], values=[1.0, 2.0], labels=[0.0, 1.0], n_cols=2), "non-decreasing"),
    (dict(indptr=[0, 2], indices=[1, 0], values=[1.0, 2.0], labels=[0.0], n_cols=2), "strictly increasing"),
    (dict(indptr=[0, 1], indices=[5], values=[1.0], labels=[0.0], n_cols=2), "out of range"),
    (dict(indptr=[0, 1], indices=[0], values=[1.0], labels=[np.inf], n_cols=1), "finite"),
    (dict(indptr=[0, 1], indices=[0], values=[1.0], labels=[0.0], n_cols=0), "n_cols"),
])
def test_invalid_csr_rejected(case, expect):
    st, h, msg = _load(np.array(case["indptr"], np.int64), np.array(case["indices"], np.int32),
                       np.array(case["values"], np.float32), np.array(case["labels"], np.float32), case["n_cols"])
    assert st == 1 and h is None and expect in msg


def test_no_cpu_fallback_without_gpu():
    try:
        import torch
        if torch.cuda.is_available():
            pytest.skip("GPU present")
    except ImportError:
        pass
    with pytest.raises(gbdt.GbdtError) as e:
        gbdt.load_csr(np.array([0, 1]), np.array([0]), np.array([1.0]), np.array([1.0]), 1)
    assert e.value.status == 3


def test_null_safe_frees():
    L = gbdt.lib()
    L.gbdt_dataset_free(None)
    L.gbdt_model_free(None)
    L.gbdt_comm_free(None)
