"""ctypes wrapper for the CPU oracle (oracle/gbdt_oracle.c). TEST INFRASTRUCTURE ONLY.

Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs may
import this module.  It shares nothing with the CUDA path; its node record is its own.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB = os.path.join(_HERE, "liboracle.so")

NODE_DTYPE = np.dtype([
    ("heap_id", np.int32), ("is_leaf", np.int32), ("attr", np.int32), ("default_left", np.int32),
    ("split_value", np.float32), ("follow_status", np.int32),
    ("gain", np.float64), ("G", np.float64), ("H", np.float64), ("weight", np.float64),
    ("count", np.int64),
], align=True)


class _Params(C.Structure):
    _fields_ = [("max_depth", C.c_int32), ("n_trees", C.c_int32), ("lam", C.c_double),
                ("gamma", C.c_double), ("eta", C.c_double), ("base_margin", C.c_double),
                ("loss", C.c_int32)]


class _Stats(C.Structure):
    _fields_ = [("nodes_exact", C.c_int64), ("nodes_near_tie", C.c_int64), ("nodes_mismatch", C.c_int64)]


def build() -> str:
    src = os.path.join(_HERE, "gbdt_oracle.c")
    if not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(src):
        subprocess.check_call(["make", "-s", "-C", _HERE])
    return _LIB


_lib = None


def lib():
    global _lib
    if _lib is None:
        _lib = C.CDLL(build())
        p = C.c_void_p
        i64 = C.c_int64
        _lib.orc_presort.restype = i64
        _lib.orc_presort.argtypes = [i64, i64, p, p, p, p, p, p]
        _lib.orc_rle_encode.restype = i64
        _lib.orc_rle_encode.argtypes = [i64, p, p, p]
        _lib.orc_seg_scan.argtypes = [i64, p, p, p]
        _lib.orc_gradients.argtypes = [C.c_int32, i64, p, p, p, p]
        _lib.orc_gain.restype = C.c_double
        _lib.orc_gain.argtypes = [C.c_double] * 5
        _lib.orc_train.restype = C.c_int
        _lib.orc_train.argtypes = [i64, i64, p, p, p, p, C.POINTER(_Params), p, p, p, C.POINTER(_Stats)]
        _lib.orc_predict.argtypes = [i64, p, p, p, p, C.c_int32, C.c_int32, C.c_double, C.c_double, p]
        _lib.orc_last_timings.restype = C.c_int
        _lib.orc_last_timings.argtypes = [p, C.c_int]
    return _lib


def _ptr(a):
    return a.ctypes.data_as(C.c_void_p) if a is not None else None


LOSS = {"squared": 0, "logistic": 1}


def presort(indptr, indices, values, n, m):
    indptr = np.ascontiguousarray(indptr, np.int64)
    indices = np.ascontiguousarray(indices, np.int32)
    values = np.ascontiguousarray(values, np.float32)
    nnz = int(indptr[-1])
    col_ptr = np.zeros(m + 1, np.int64)
    val = np.zeros(max(nnz, 1), np.float32)
    ins = np.zeros(max(nnz, 1), np.int32)
    k = lib().orc_presort(n, m, _ptr(indptr), _ptr(indices), _ptr(values), _ptr(col_ptr), _ptr(val), _ptr(ins))
    return col_ptr, val[:k], ins[:k]


def rle_encode(vals):
    vals = np.ascontiguousarray(vals, np.float32)
    rv = np.zeros(max(vals.size, 1), np.float32)
    rl = np.zeros(max(vals.size, 1), np.int32)
    r = lib().orc_rle_encode(vals.size, _ptr(vals), _ptr(rv), _ptr(rl))
    return rv[:r], rl[:r]


def seg_scan(x, head):
    x = np.ascontiguousarray(x, np.float64)
    head = np.ascontiguousarray(head, np.uint8)
    out = np.zeros_like(x)
    lib().orc_seg_scan(x.size, _ptr(x), _ptr(head), _ptr(out))
    return out


def gradients(loss, yhat, y):
    yhat = np.ascontiguousarray(yhat, np.float64)
    y = np.ascontiguousarray(y, np.float32)
    g = np.zeros_like(yhat)
    h = np.zeros_like(yhat)
    lib().orc_gradients(LOSS[loss], yhat.size, _ptr(yhat), _ptr(y), _ptr(g), _ptr(h))
    return g, h


def gain(GL, HL, G, H, lam):
    return lib().orc_gain(GL, HL, G, H, lam)


def train(prob, params=None, follow=None):
    """Returns (nodes[T, 2^(d+1)-1] structured array, margin[n], stats dict)."""
    P = dict(prob.params)
    if params:
        P.update(params)
    d, T = int(P["max_depth"]), int(P["n_trees"])
    NH = (1 << (d + 1)) - 1
    prm = _Params(d, T, float(P["lam"]), float(P["gamma"]), float(P["eta"]),
                  float(P.get("base_margin", 0.0)), LOSS[P["loss"]])
    nodes = np.zeros((T, NH), NODE_DTYPE)
    margin = np.zeros(prob.n, np.float64)
    st = _Stats()
    fol = None
    if follow is not None:
        fol = np.zeros((T, NH), NODE_DTYPE)
        for f in follow.dtype.names:
            if f in NODE_DTYPE.names:
                fol[f] = follow[f]
    indptr = np.ascontiguousarray(prob.indptr, np.int64)
    indices = np.ascontiguousarray(prob.indices, np.int32)
    values = np.ascontiguousarray(prob.values, np.float32)
    labels = np.ascontiguousarray(prob.labels, np.float32)
    rc = lib().orc_train(prob.n, prob.m, _ptr(indptr), _ptr(indices), _ptr(values), _ptr(labels),
                         C.byref(prm), _ptr(fol), _ptr(nodes), _ptr(margin), C.byref(st))
    if rc != 0:
        raise ValueError(f"orc_train failed ({rc})")
    return nodes, margin, dict(exact=st.nodes_exact, near_tie=st.nodes_near_tie, mismatch=st.nodes_mismatch)


def last_timings():
    """Wall-clock seconds of the calling thread's last train(): (presort_s, [tree_s, ...])."""
    buf = np.zeros(4097, np.float64)
    k = min(lib().orc_last_timings(_ptr(buf), buf.size), buf.size)
    return float(buf[0]), buf[1:k].tolist()


def predict(nodes, indptr, indices, values, eta, base_margin=0.0):
    T, NH = nodes.shape
    d = int(np.log2(NH + 1)) - 1
    indptr = np.ascontiguousarray(indptr, np.int64)
    n = indptr.size - 1
    indices = np.ascontiguousarray(indices, np.int32)
    values = np.ascontiguousarray(values, np.float32)
    nodes = np.ascontiguousarray(nodes, NODE_DTYPE)
    out = np.zeros(n, np.float64)
    lib().orc_predict(n, _ptr(indptr), _ptr(indices), _ptr(values), _ptr(nodes), T, d,
                      float(eta), float(base_margin), _ptr(out))
    return out
