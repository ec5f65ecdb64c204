"""Thin ctypes binding of libgbdt.so (include/gbdt.h).  Argument marshalling only: every step of
training and prediction runs in the library's CUDA kernels.  There is no CPU fallback -- if the
shared library is missing or no CUDA device is usable, calls raise.

Function names follow the C ABI: load_csr, train, predict, comm_unique_id, comm_init.
PyTorch is used only to obtain the current CUDA stream and, for multi-process sharding, to
broadcast the NCCL unique id over torch.distributed.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
# GBDT_LIB: an alternative in-tree build of the same library (A/B measurements of kernel variants)
LIB_PATH = os.environ.get("GBDT_LIB") or os.path.join(_HERE, "libgbdt.so")

GBDT_OK = 0
STATUS = {0: "OK", 1: "E_INVAL", 2: "E_NOMEM", 3: "E_CUDA", 4: "E_NCCL", 5: "E_STATE", 6: "E_RANGE"}
LOSS = {"squared": 0, "logistic": 1, "custom": 2}
RLE = {"off": 0, "on": 1, "auto": 2, False: 0, True: 1, None: 0}
PHASES = ["grad", "split_find", "decide", "nodemap", "partition", "comm", "total",
          "k_chunk_agg", "k_split", "k_count", "k_scatter", "k_fused"]

NODE_DTYPE = np.dtype([
    ("heap_id", np.int32), ("is_leaf", np.int32), ("attr", np.int32), ("default_left", np.int32),
    ("split_value", np.float32), ("reserved", np.int32),
    ("gain", np.float64), ("G", np.float64), ("H", np.float64), ("weight", np.float64),
    ("count", np.int64),
])
assert NODE_DTYPE.itemsize == 64


class GbdtError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"{STATUS.get(status, status)}: {msg}")
        self.status = status


class _LoadOpts(C.Structure):
    _fields_ = [("rle", C.c_int32), ("rle_min_ratio", C.c_double), ("n_shards", C.c_int32),
                ("device", C.c_int32), ("stream", C.c_void_p), ("comm", C.c_void_p), ("keep_rows", C.c_int32),
                ("dense", C.c_int32), ("dense_fill", C.c_float)]


# gbdt_grad_fn(n, yhat, labels, g, h, stream, user): device pointers (GBDT_LOSS_CUSTOM)
GRAD_FN = C.CFUNCTYPE(C.c_int, C.c_int64, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p, C.c_void_p)


class _Params(C.Structure):
    _fields_ = [("max_depth", C.c_int32), ("n_trees", C.c_int32), ("lam", C.c_double),
                ("gamma", C.c_double), ("eta", C.c_double), ("base_margin", C.c_double),
                ("loss", C.c_int32), ("profile", C.c_int32), ("smartgd_off", C.c_int32),
                ("rle_decompress", C.c_int32), ("grad_fn", GRAD_FN), ("grad_user", C.c_void_p)]


_lib = None


def lib():
    """Loads the in-tree libgbdt.so; raises if it has not been built."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = C.CDLL(LIB_PATH)
    p, i32, i64 = C.c_void_p, C.c_int32, C.c_int64
    L.gbdt_last_error.restype = C.c_char_p
    L.gbdt_last_launch_count.restype = C.c_int64
    L.gbdt_load_csr.argtypes = [i64, i64, p, p, p, p, C.POINTER(_LoadOpts), C.POINTER(p)]
    L.gbdt_train.argtypes = [p, C.POINTER(_Params), C.POINTER(p), p]
    L.gbdt_predict.argtypes = [p, i64, i64, p, p, p, i32, p]
    L.gbdt_predict_on_stream.argtypes = [p, i64, i64, p, p, p, i32, p, p]
    L.gbdt_model_train_loss.argtypes = [p, p]
    L.gbdt_model_export_level.argtypes = [p, i32] + [p] * 11
    L.gbdt_model_num_trees.argtypes = [p, C.POINTER(i32)]
    L.gbdt_model_num_nodes.argtypes = [p, i32, C.POINTER(i32)]
    L.gbdt_model_export.argtypes = [p, i32, p]
    L.gbdt_get_timings.argtypes = [p, p, i32]
    L.gbdt_get_level_entries.argtypes = [p, p, i32]
    L.gbdt_dataset_info.argtypes = [p, i32, p]
    L.gbdt_dataset_export_layout.argtypes = [p, i32, p, p, p]
    L.gbdt_dataset_export_rle.argtypes = [p, i32, p, p, p]
    L.gbdt_comm_unique_id.argtypes = [p]
    L.gbdt_comm_init.argtypes = [i32, i32, p, i32, C.POINTER(p)]
    L.gbdt_comm_free.argtypes = [p]
    L.gbdt_comm_init_callbacks.argtypes = [i32, i32, _AG_FN, _AR_FN, p, i32, C.POINTER(p)]
    L.gbdt_shard_ranges.argtypes = [i64, p, i32, p]
    L.gbdt_dataset_free.argtypes = [p]
    L.gbdt_model_free.argtypes = [p]
    for f in ("gbdt_load_csr", "gbdt_train", "gbdt_predict", "gbdt_predict_on_stream", "gbdt_model_train_loss",
              "gbdt_model_export_level",
              "gbdt_model_num_trees", "gbdt_model_num_nodes",
              "gbdt_model_export", "gbdt_get_timings", "gbdt_get_level_entries", "gbdt_dataset_info", "gbdt_dataset_export_layout",
              "gbdt_dataset_export_rle", "gbdt_comm_unique_id", "gbdt_comm_init", "gbdt_comm_init_callbacks",
              "gbdt_shard_ranges"):
        getattr(L, f).restype = C.c_int
    _lib = L
    return L


def _check(st):
    if st != GBDT_OK:
        raise GbdtError(st, lib().gbdt_last_error().decode())


def _p(a):
    return None if a is None else a.ctypes.data_as(C.c_void_p)


def _current_stream():
    try:
        import torch
        if torch.cuda.is_available():
            return torch.cuda.current_stream().cuda_stream
    except Exception:
        pass
    return None


def last_launch_count() -> int:
    return int(lib().gbdt_last_launch_count())


_AG_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_void_p, C.c_size_t, C.c_void_p)
_AR_FN = C.CFUNCTYPE(C.c_int, C.c_void_p, C.c_size_t, C.c_void_p)


class Comm:
    """NCCL communicator (one process per GPU).  Use :func:`comm_from_torch` under torchrun."""

    def __init__(self, handle, keep=None):
        self._h = handle
        self._keep = keep  # callback trampolines must outlive the handle

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.gbdt_comm_free(self._h)
            self._h = None


def comm_unique_id() -> bytes:
    buf = (C.c_uint8 * 128)()
    _check(lib().gbdt_comm_unique_id(C.cast(buf, C.c_void_p)))
    return bytes(buf)


def comm_init(rank: int, world: int, uid: bytes, device: int = -1) -> Comm:
    buf = (C.c_uint8 * 128).from_buffer_copy(uid)
    h = C.c_void_p()
    _check(lib().gbdt_comm_init(rank, world, C.cast(buf, C.c_void_p), device, C.byref(h)))
    return Comm(h)


def shard_ranges(col_counts, P: int) -> np.ndarray:
    """Attribute ranges [b[i], b[i+1]) of a P-way sharding balanced by entries (host only)."""
    cc = np.ascontiguousarray(col_counts, np.int64)
    b = np.zeros(P + 1, np.int32)
    _check(lib().gbdt_shard_ranges(cc.size, _p(cc), int(P), _p(b)))
    return b


def torch_collectives(group=None):
    """(allgather, allreduce_u8) over host buffers given as addresses, run on a torch.distributed
    group; the callbacks of :func:`comm_from_callbacks` (return 0 on success)."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)

    def ag(send, recv, nbytes, user):
        try:
            src = torch.frombuffer((C.c_uint8 * nbytes).from_address(send), dtype=torch.uint8).clone()
            out = torch.empty(nbytes * world, dtype=torch.uint8)
            dist.all_gather_into_tensor(out, src, group=group)
            C.memmove(recv, out.numpy().ctypes.data, nbytes * world)
            return 0
        except Exception:  # noqa: BLE001 - reported to the library as a failed collective
            return 1

    def ar(buf, n, user):
        try:
            t = torch.frombuffer((C.c_uint8 * n).from_address(buf), dtype=torch.uint8).to(torch.int32)
            dist.all_reduce(t, group=group)
            res = t.to(torch.uint8).numpy()  # keep alive across the copy
            C.memmove(buf, res.ctypes.data, n)
            return 0
        except Exception:  # noqa: BLE001
            return 1

    return ag, ar


def comm_from_callbacks(device: int = -1, group=None) -> Comm:
    """Host-staged communicator whose collectives run over a torch.distributed group (e.g.
    gloo).  For tests of the sharded path where NCCL cannot run (several ranks on one GPU)."""
    import torch.distributed as dist
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    ag, ar = torch_collectives(group)
    fa, fr = _AG_FN(ag), _AR_FN(ar)
    h = C.c_void_p()
    _check(lib().gbdt_comm_init_callbacks(rank, world, fa, fr, None, device, C.byref(h)))
    return Comm(h, keep=(fa, fr))


def comm_from_torch(device: int = -1) -> Comm:
    """Bootstraps the NCCL id through the default torch.distributed process group."""
    import torch
    import torch.distributed as dist
    rank, world = dist.get_rank(), dist.get_world_size()
    uid = comm_unique_id() if rank == 0 else bytes(128)
    t = torch.tensor(list(uid), dtype=torch.uint8)
    if dist.get_backend() == "nccl":
        t = t.cuda()
    dist.broadcast(t, 0)
    return comm_init(rank, world, bytes(t.cpu().tolist()), device)


class Dataset:
    def __init__(self, handle, n, m, keep):
        self._h = handle
        self.n, self.m = n, m
        self._keep = keep

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.gbdt_dataset_free(self._h)
            self._h = None

    def info(self, shard=0):
        a = np.zeros(7, np.int64)
        _check(lib().gbdt_dataset_info(self._h, shard, _p(a)))
        return dict(n=int(a[0]), m=int(a[1]), nnz=int(a[2]), n_shards=int(a[3]), attr_begin=int(a[4]),
                    attr_end=int(a[5]), runs=int(a[6]))

    def export_layout(self, shard=0):
        inf = self.info(shard)
        ms = inf["attr_end"] - inf["attr_begin"]
        col_ptr = np.zeros(ms + 1, np.int64)
        val = np.zeros(max(inf["nnz"], 1), np.float32)
        ins = np.zeros(max(inf["nnz"], 1), np.int32)
        _check(lib().gbdt_dataset_export_layout(self._h, shard, _p(col_ptr), _p(val), _p(ins)))
        return col_ptr, val[:inf["nnz"]], ins[:inf["nnz"]]

    def export_rle(self, shard=0):
        inf = self.info(shard)
        ms = inf["attr_end"] - inf["attr_begin"]
        run_ptr = np.zeros(ms + 1, np.int64)
        R = max(inf["runs"], 1)
        rv = np.zeros(R, np.float32)
        rl = np.zeros(R, np.int32)
        _check(lib().gbdt_dataset_export_rle(self._h, shard, _p(run_ptr), _p(rv), _p(rl)))
        return run_ptr, rv[:inf["runs"]], rl[:inf["runs"]]


class Model:
    def __init__(self, handle):
        self._h = handle

    def __del__(self):
        if getattr(self, "_h", None) and _lib is not None:
            _lib.gbdt_model_free(self._h)
            self._h = None

    @property
    def n_trees(self):
        v = C.c_int32()
        _check(lib().gbdt_model_num_trees(self._h, C.byref(v)))
        return v.value

    def nodes(self) -> np.ndarray:
        """All trees, heap order: array of shape (n_trees, 2^(d+1)-1) with NODE_DTYPE."""
        T = self.n_trees
        v = C.c_int32()
        _check(lib().gbdt_model_num_nodes(self._h, 0, C.byref(v)))
        out = np.zeros((T, v.value), NODE_DTYPE)
        for t in range(T):
            row = np.zeros(v.value, NODE_DTYPE)
            _check(lib().gbdt_model_export(self._h, t, _p(row)))
            out[t] = row
        return out

    def export_level(self, shard=0) -> dict:
        """The level captured with GBDT_CAPTURE_LEVEL (test hook; see gbdt_model_export_level)."""
        info = np.zeros(5, np.int64)
        L = lib()
        N = None
        _check(L.gbdt_model_export_level(self._h, shard, _p(info), N, N, N, N, N, N, N, N, N, N))
        m, K, n, R = int(info[1]), int(info[2]), int(info[3]), int(info[4])
        out = dict(shard=int(info[0]), m=m, K=K, col_start=np.zeros(m + 1, np.int64), col_len=np.zeros(m, np.int64),
                   seg_start=np.zeros(m * K, np.int64), seg_cnt=np.zeros(m * K, np.int64),
                   val=np.zeros(n, np.float32), ins=np.zeros(n, np.int32), run_val=np.zeros(R, np.float32),
                   run_len=np.zeros(R, np.int32), run_pos=np.zeros(R, np.int64),
                   seg_run=np.zeros(m * K + 1 if R else 0, np.int32))
        _check(L.gbdt_model_export_level(self._h, shard, _p(info), *[_p(out[k]) for k in (
            "col_start", "col_len", "seg_start", "seg_cnt", "val", "ins", "run_val", "run_len", "run_pos", "seg_run")]))
        return out

    def train_loss(self) -> np.ndarray:
        """Mean training loss after 0 .. T trees (squared: (y-yhat)^2, RMSE = sqrt; logistic: log loss)."""
        a = np.zeros(self.n_trees + 1, np.float64)
        _check(lib().gbdt_model_train_loss(self._h, _p(a)))
        return a

    def timings(self) -> dict:
        a = np.zeros(len(PHASES), np.float64)
        _check(lib().gbdt_get_timings(self._h, _p(a), len(PHASES)))
        return dict(zip(PHASES, a.tolist()))

    def level_entries(self, levels: int) -> np.ndarray:
        """List entries split finding scanned per level, summed over the trees (profile=True)."""
        a = np.zeros(levels, np.int64)
        _check(lib().gbdt_get_level_entries(self._h, _p(a), levels))
        return a

    def predict(self, indptr, indices, values, n_cols, output_margin=True) -> np.ndarray:
        return predict(self, indptr, indices, values, n_cols, output_margin)


def load_csr(indptr, indices, values, labels, n_cols, rle="off", rle_min_ratio=0.0, n_shards=1,
             device=-1, stream="current", comm: Comm | None = None, keep_rows=False, dense=False,
             dense_fill=0.0) -> Dataset:
    indptr = np.ascontiguousarray(indptr, np.int64)
    indices = np.ascontiguousarray(indices, np.int32)
    values = np.ascontiguousarray(values, np.float32)
    labels = np.ascontiguousarray(labels, np.float32)
    n = indptr.size - 1
    if stream == "current":
        stream = _current_stream()
    o = _LoadOpts(RLE[rle], float(rle_min_ratio), int(n_shards), int(device), stream,
                  comm._h if comm is not None else None, int(bool(keep_rows)), int(bool(dense)), float(dense_fill))
    h = C.c_void_p()
    _check(lib().gbdt_load_csr(n, int(n_cols), _p(indptr), _p(indices), _p(values), _p(labels), C.byref(o),
                               C.byref(h)))
    return Dataset(h, n, int(n_cols), None)


def train(ds: Dataset, max_depth=6, n_trees=40, lam=1.0, gamma=0.0, eta=0.3, base_margin=0.0,
          loss="squared", profile=False, want_margin=True, smartgd=True, grad_fn=None, rle_split="direct"):
    """grad_fn (loss="custom"): python callable (n, yhat, labels, g, h, stream) -> None over
    DEVICE addresses, run on the library's stream (see gbdt_grad_fn in include/gbdt.h).
    rle_split: "direct" (Fig. 7) or "decompress" (the P:248 / Fig. 6 ablation)."""
    cb = GRAD_FN()
    if grad_fn is not None:
        def _tramp(n, yh, y, g, h, st, user):
            try:
                grad_fn(int(n), yh, y, g, h, st)
                return 0
            except Exception:  # noqa: BLE001 - reported to the library as a failed callback
                import traceback
                traceback.print_exc()
                return 1
        cb = GRAD_FN(_tramp)
    prm = _Params(int(max_depth), int(n_trees), float(lam), float(gamma), float(eta), float(base_margin),
                  LOSS[loss], int(bool(profile)), int(not smartgd), {"direct": 0, "decompress": 1}[rle_split], cb, None)
    h = C.c_void_p()
    margin = np.zeros(ds.n, np.float64) if want_margin else None
    _check(lib().gbdt_train(ds._h, C.byref(prm), C.byref(h), _p(margin)))
    return Model(h), margin


def predict(model: Model, indptr, indices, values, n_cols, output_margin=True, stream="current") -> np.ndarray:
    indptr = np.ascontiguousarray(indptr, np.int64)
    indices = np.ascontiguousarray(indices, np.int32)
    values = np.ascontiguousarray(values, np.float32)
    n = indptr.size - 1
    out = np.zeros(n, np.float64)
    if stream == "current":
        stream = _current_stream()
    _check(lib().gbdt_predict_on_stream(model._h, n, int(n_cols), _p(indptr), _p(indices), _p(values),
                                        int(bool(output_margin)), _p(out), stream))
    return out


def train_problem(prob, **overrides):
    """Convenience: load + train a datagen.synth.Problem with its own parameters."""
    P = dict(prob.params)
    P.update(overrides)
    rle = P.pop("rle", "off")
    n_shards = P.pop("n_shards", 1)
    dense = P.pop("dense", False)
    dense_fill = P.pop("dense_fill", 0.0)
    keep_rows = not P.get("smartgd", True)  # the SmartGD-off ablation traverses the CSR rows
    ds = load_csr(prob.indptr, prob.indices, prob.values, prob.labels, prob.m, rle=rle, n_shards=n_shards,
                  keep_rows=keep_rows, dense=dense, dense_fill=dense_fill)
    return train(ds, **P)
