// api.cpp -- the C ABI of libgbdt.so (include/gbdt.h): validation, handles, error reporting.
#include <cmath>
#include <atomic>
#include <climits>
#include <cstring>
#include <thread>
#include <exception>
#include <algorithm>
#include <limits>
#include <mutex>
#include <new>
#include <string>
#include <vector>

#include "internal.h"

namespace gbdt {

namespace {
thread_local std::string g_err;
}

void fail(gbdt_status st, const std::string& msg) { throw Error{st, msg}; }

// The library's own stream-ordered memory pool per device: freed allocations stay cached in it
// across gbdt_train / gbdt_load_csr calls (release threshold = max), without touching the
// process-wide default pool that other libraries (PyTorch) allocate from.
static cudaMemPool_t lib_pool(int dev) {
  static std::once_flag once[kMaxDevices];
  static cudaMemPool_t pools[kMaxDevices];
  static cudaError_t errs[kMaxDevices];
  if (dev < 0 || dev >= kMaxDevices) fail(GBDT_E_RANGE, "device ordinal >= " + std::to_string(kMaxDevices));
  std::call_once(once[dev], [dev] {
    cudaMemPoolProps props;
    std::memset(&props, 0, sizeof props);
    props.allocType = cudaMemAllocationTypePinned;
    props.handleTypes = cudaMemHandleTypeNone;
    props.location.type = cudaMemLocationTypeDevice;
    props.location.id = dev;
    errs[dev] = cudaMemPoolCreate(&pools[dev], &props);
    if (errs[dev] == cudaSuccess) {
      uint64_t thr = UINT64_MAX;
      errs[dev] = cudaMemPoolSetAttribute(pools[dev], cudaMemPoolAttrReleaseThreshold, &thr);
    }
  });
  GBDT_CUDA(errs[dev]);
  return pools[dev];
}

void DBuf::alloc(size_t b, cudaStream_t s) {
  release();
  st = s;
  bytes = b ? b : 16;
  int dev = 0;
  GBDT_CUDA(cudaGetDevice(&dev));
  GBDT_CUDA(cudaMallocFromPoolAsync(&p, bytes, lib_pool(dev), st));
}

void DBuf::release() {
  if (p) {
    cudaFreeAsync(p, st);
    p = nullptr;
    bytes = 0;
  }
}

int64_t launches_get();
void comm_unique_id(uint8_t id[128]);
Comm* comm_init(int rank, int world, const uint8_t id[128], int device);
void comm_free(Comm* c);

template <class F>
static gbdt_status guarded(F&& f) {
  try {
    g_err.clear();
    f();
    return GBDT_OK;
  } catch (const Error& e) {
    g_err = e.msg;
    return e.st;
  } catch (const std::bad_alloc&) {
    g_err = "host allocation failed";
    return GBDT_E_NOMEM;
  } catch (const std::exception& e) {
    g_err = e.what();
    return GBDT_E_CUDA;
  }
}

// Runs f(lo, hi) over [0, n) split into contiguous ranges on up to hardware_concurrency threads
// (one range when n is small).
template <class F>
static void parallel_ranges(int64_t n, int64_t min_per_thread, F&& f) {
  const int64_t hw = std::max<int64_t>(1, (int64_t)std::thread::hardware_concurrency());
  const int64_t T = std::max<int64_t>(1, std::min<int64_t>(std::min<int64_t>(hw, 64), n / std::max<int64_t>(min_per_thread, 1)));
  if (T == 1) { f(0, n, 0); return; }
  std::vector<std::thread> th;
  for (int64_t t = 0; t < T; ++t) th.emplace_back([&, t] { f(n * t / T, n * (t + 1) / T, (int)t); });
  for (auto& x : th) x.join();
}

// CSR structure checks shared by load and predict (P:32 sparse rows; indices strictly increasing).
// Row ranges are checked in parallel; the error reported is the one of the first bad row, as a
// sequential scan would report it.
static void validate_csr(int64_t n_rows, int64_t n_cols, const int64_t* indptr, const int32_t* indices,
                         const float* values, bool require_cols_in_range) {
  const int64_t kMax = (int64_t(1) << 31) - 1;
  if (n_rows < 1 || n_rows >= kMax) fail(GBDT_E_INVAL, "n_rows must be in [1, 2^31-1)");
  if (n_cols < 1 || n_cols >= kMax) fail(GBDT_E_INVAL, "n_cols must be in [1, 2^31-1)");
  if (!indptr) fail(GBDT_E_INVAL, "indptr is NULL");
  if (indptr[0] != 0) fail(GBDT_E_INVAL, "indptr[0] must be 0");
  std::atomic<int64_t> bad{INT64_MAX};
  auto note = [&](int64_t i) {
    int64_t cur = bad.load();
    while (i < cur && !bad.compare_exchange_weak(cur, i)) {
    }
  };
  parallel_ranges(n_rows, 1 << 16, [&](int64_t lo, int64_t hi, int) {
    for (int64_t i = lo; i < hi; ++i)
      if (indptr[i + 1] < indptr[i]) { note(i); return; }
  });
  if (bad.load() != INT64_MAX)
    fail(GBDT_E_INVAL, "indptr must be non-decreasing (row " + std::to_string(bad.load()) + ")");
  const int64_t nnz = indptr[n_rows];
  if (nnz >= kMax) fail(GBDT_E_INVAL, "nnz must be < 2^31-1");
  if (nnz > 0 && (!indices || !values)) fail(GBDT_E_INVAL, "indices/values NULL with nnz > 0");
  std::vector<int> kind(64, 0);  // per thread: 1 out of range, 2 not increasing (at its first bad row)
  std::vector<int64_t> first(64, INT64_MAX);
  parallel_ranges(n_rows, 1 << 14, [&](int64_t lo, int64_t hi, int t) {
    for (int64_t i = lo; i < hi; ++i) {
      int32_t prev = -1;
      for (int64_t p = indptr[i]; p < indptr[i + 1]; ++p) {
        const int32_t a = indices[p];
        if (a < 0 || (require_cols_in_range && a >= n_cols)) { kind[t] = 1; first[t] = i; return; }
        if (a <= prev) { kind[t] = 2; first[t] = i; return; }
        prev = a;
      }
    }
  });
  int bt = -1;
  for (int t = 0; t < 64; ++t)
    if (kind[t] && (bt < 0 || first[t] < first[bt])) bt = t;
  if (bt >= 0) {
    if (kind[bt] == 1) fail(GBDT_E_INVAL, "column index out of range in row " + std::to_string(first[bt]));
    fail(GBDT_E_INVAL, "column indices must be strictly increasing in row " + std::to_string(first[bt]));
  }
}

}  // namespace gbdt

using namespace gbdt;

struct gbdt_dataset {
  Dataset ds;
};
struct gbdt_model {
  Model m;
};
struct gbdt_comm {
  Comm* c = nullptr;
};

namespace gbdt {
std::vector<int32_t> shard_ranges(int64_t n_cols, const int64_t* col_counts, int P) {
  std::vector<int64_t> pre(n_cols + 1, 0);
  for (int64_t a = 0; a < n_cols; ++a) pre[a + 1] = pre[a] + col_counts[a];
  std::vector<int32_t> bnd(P + 1, 0);
  bnd[P] = (int32_t)n_cols;
  int64_t a = 0;
  for (int i = 1; i < P; ++i) {
    const double target = (double)pre[n_cols] * i / P;
    while (a < n_cols && (double)pre[a] < target) ++a;
    bnd[i] = (int32_t)std::max<int64_t>(a, bnd[i - 1]);
  }
  return bnd;
}
}  // namespace gbdt

extern "C" {

const char* gbdt_last_error(void) { return g_err.c_str(); }

int64_t gbdt_last_launch_count(void) { return launches_get(); }

gbdt_status gbdt_load_csr(int64_t n_rows, int64_t n_cols, const int64_t* indptr, const int32_t* indices,
                          const float* values, const float* labels, const gbdt_load_opts* opts,
                          gbdt_dataset** out) {
  if (out) *out = nullptr;
  return guarded([&] {
    if (!out) fail(GBDT_E_INVAL, "out is NULL");
    float lmin = std::numeric_limits<float>::infinity(), lmax = -lmin;
    bool binary = true;
    // the full O(nnz) checks: run on the host cores while the H2D copies are in flight
    auto validate_all = [&] {
      validate_csr(n_rows, n_cols, indptr, indices, values, true);
      if (!labels) fail(GBDT_E_INVAL, "labels is NULL");
      struct LabelStats { float lo, hi; bool bin; int64_t bad; };
      std::vector<LabelStats> ls(64, LabelStats{lmin, lmax, true, INT64_MAX});
      parallel_ranges(n_rows, 1 << 16, [&](int64_t lo, int64_t hi, int t) {
        LabelStats& L = ls[t];
        for (int64_t i = lo; i < hi; ++i) {
          const float y = labels[i];
          if (!std::isfinite(y)) { L.bad = i; return; }
          L.bin &= (y == 0.0f || y == 1.0f);
          L.lo = std::min(L.lo, y);
          L.hi = std::max(L.hi, y);
        }
      });
      int64_t bad = INT64_MAX;
      for (const LabelStats& L : ls) {
        bad = std::min(bad, L.bad);
        binary &= L.bin;
        lmin = std::min(lmin, L.lo);
        lmax = std::max(lmax, L.hi);
      }
      if (bad != INT64_MAX) fail(GBDT_E_INVAL, "labels must be finite (row " + std::to_string(bad) + ")");
    };
    // O(1) checks needed before anything is copied
    const int64_t kMax = (int64_t(1) << 31) - 1;
    if (n_rows < 1 || n_rows >= kMax) fail(GBDT_E_INVAL, "n_rows must be in [1, 2^31-1)");
    if (n_cols < 1 || n_cols >= kMax) fail(GBDT_E_INVAL, "n_cols must be in [1, 2^31-1)");
    if (!indptr) fail(GBDT_E_INVAL, "indptr is NULL");
    if (indptr[0] != 0) fail(GBDT_E_INVAL, "indptr[0] must be 0");
    gbdt_load_opts o;
    std::memset(&o, 0, sizeof o);
    if (opts) o = *opts;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || ndev < 1) {
      validate_all();  // argument errors are reported before the missing device
      fail(GBDT_E_CUDA, "no CUDA device visible");
    }
    if (indptr[n_rows] < 0 || indptr[n_rows] >= kMax || !labels ||
        (indptr[n_rows] > 0 && (!indices || !values))) {
      validate_all();  // reports the precise error
      fail(GBDT_E_INVAL, "malformed CSR");
    }
    if (o.rle < 0 || o.rle > 2) fail(GBDT_E_INVAL, "rle must be OFF, ON or AUTO");
    int nsh = o.n_shards <= 0 ? 1 : o.n_shards;
    if (nsh != 1 && nsh != 2 && nsh != 4 && nsh != 8) fail(GBDT_E_RANGE, "n_shards must be 1, 2, 4 or 8");
    Comm* comm = o.comm ? o.comm->c : nullptr;
    if (comm && nsh != 1) fail(GBDT_E_RANGE, "n_shards must be 1 with a communicator");
    int dev = o.device;
    if (dev < 0) GBDT_CUDA(cudaGetDevice(&dev));
    if (dev >= ndev) fail(GBDT_E_RANGE, "device ordinal out of range");
    if (comm) dev = comm->device;
    GBDT_CUDA(cudaSetDevice(dev));

    const int64_t nnz = indptr[n_rows];

    auto* h = new gbdt_dataset();
    Dataset& ds = h->ds;
    try {
      cudaStream_t st = (cudaStream_t)o.stream;
      DBuf dptr((size_t)(n_rows + 1) * 8, st), didx((size_t)std::max<int64_t>(nnz, 1) * 4, st),
          dval((size_t)std::max<int64_t>(nnz, 1) * 4, st);
      GBDT_CUDA(cudaMemcpyAsync(dptr.p, indptr, (size_t)(n_rows + 1) * 8, cudaMemcpyHostToDevice, st));
      if (nnz) {
        GBDT_CUDA(cudaMemcpyAsync(didx.p, indices, (size_t)nnz * 4, cudaMemcpyHostToDevice, st));
        GBDT_CUDA(cudaMemcpyAsync(dval.p, values, (size_t)nnz * 4, cudaMemcpyHostToDevice, st));
      }
      ds.y.alloc((size_t)n_rows * 4, st);
      GBDT_CUDA(cudaMemcpyAsync(ds.y.p, labels, (size_t)n_rows * 4, cudaMemcpyHostToDevice, st));
      try {
        validate_all();  // overlaps the copies (from pinned host memory they run asynchronously)
      } catch (...) {
        cudaStreamSynchronize(st);  // the copies still read the caller's buffers
        throw;
      }
      int64_t nnz_l = nnz;
      if (o.dense) {  // dense representation: the filled matrix replaces the CSR
        if (!std::isfinite(o.dense_fill)) fail(GBDT_E_INVAL, "dense_fill must be finite");
        if ((double)n_rows * (double)n_cols >= (double)kMax) fail(GBDT_E_RANGE, "dense matrix exceeds 2^31 - 1 entries");
        DBuf fptr, fidx, fval;
        densify(n_rows, n_cols, dptr.as<int64_t>(), didx.as<int32_t>(), dval.as<float>(), o.dense_fill, fptr, fidx,
                fval, st);
        dptr = std::move(fptr);
        didx = std::move(fidx);
        dval = std::move(fval);
        nnz_l = n_rows * n_cols;
      }
      // present entries per attribute, counted on the device
      const std::vector<int64_t> col_counts = column_counts(nnz_l, n_cols, didx.as<int32_t>(), dval.as<float>(), st);
      bool missing = false;
      for (int64_t a = 0; a < n_cols; ++a) missing |= col_counts[a] != n_rows;
      ds.n = n_rows;
      ds.m = n_cols;
      ds.nnz = nnz_l;
      ds.dense = o.dense ? 1 : 0;
      ds.fill = o.dense ? o.dense_fill : 0.f;
      ds.device = dev;
      ds.stream = st;
      ds.has_missing = missing;
      ds.binary_labels = binary;
      ds.comm = comm;
      ds.rle = o.rle;
      ds.h_labels_minmax = {lmin, lmax};
      const int world = comm ? comm->world : 1;
      int P = comm ? world : nsh;
      // contiguous attribute ranges balanced by stored entries
      std::vector<int32_t> bnd = shard_ranges(n_cols, col_counts.data(), P);
      if (o.rle == GBDT_RLE_AUTO && !comm && nsh == 1) {
        // AUTO per attribute (reading R21 of P:237, "dimensionality / cardinality > R"): attribute a
        // is compressed iff entries_a / runs_a >= rle_min_ratio.  The runs are counted on an
        // uncompressed layout; the attributes are then regrouped into shards of equal decision
        // (maximal contiguous ranges; trees are identical for any attribute sharding), and each
        // shard's aggregate ratio falls on the same side of the threshold as its attributes.
        ds.rle = GBDT_RLE_OFF;
        ds.n_total_shards = 1;
        auto probe = std::make_unique<Shard>();
        probe->index = 0; probe->a_begin = 0; probe->a_end = (int32_t)n_cols; probe->m = (int32_t)n_cols;
        ds.shards.push_back(std::move(probe));
        build_layout(ds, dptr.as<int64_t>(), didx.as<int32_t>(), dval.as<float>(), col_counts, o.rle_min_ratio);
        int sms = 148;
        GBDT_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
        const std::vector<uint32_t> runs = attribute_runs(*ds.shards[0], st, sms);
        ds.shards.clear();
        const double thr = o.rle_min_ratio > 0 ? o.rle_min_ratio : 2.0;
        std::vector<int32_t> groups{0};
        int prev = -1;
        for (int64_t a = 0; a < n_cols; ++a) {
          const int dcs = runs[a] > 0 && (double)col_counts[a] >= thr * (double)runs[a];
          if (a > 0 && dcs != prev) groups.push_back((int32_t)a);
          prev = dcs;
        }
        groups.push_back((int32_t)n_cols);
        if (groups.size() - 1 <= 64) {  // else: many alternations, keep the entry-balanced single shard
          bnd = groups;
          P = (int)groups.size() - 1;
        }
        ds.rle = GBDT_RLE_AUTO;
      }
      ds.n_total_shards = P;
      for (int i = 0; i < P; ++i) {
        if (comm && i != comm->rank) continue;
        auto sh = std::make_unique<Shard>();
        sh->index = i;
        sh->a_begin = bnd[i];
        sh->a_end = bnd[i + 1];
        sh->m = sh->a_end - sh->a_begin;
        ds.shards.push_back(std::move(sh));
      }
      build_layout(ds, dptr.as<int64_t>(), didx.as<int32_t>(), dval.as<float>(), col_counts, o.rle_min_ratio);
      if (o.keep_rows) {
        ds.rows_ptr = std::move(dptr);
        ds.rows_idx = std::move(didx);
        ds.rows_val = std::move(dval);
      } else {
        dptr.release();
        didx.release();
        dval.release();
      }
      GBDT_CUDA(cudaStreamSynchronize(st));
    } catch (...) {
      delete h;
      throw;
    }
    *out = h;
  });
}

gbdt_status gbdt_train(gbdt_dataset* dsh, const gbdt_params* p, gbdt_model** out, double* train_margin) {
  if (out) *out = nullptr;
  return guarded([&] {
    if (!dsh || !p || !out) fail(GBDT_E_INVAL, "NULL argument");
    Dataset& ds = dsh->ds;
    if (p->max_depth < 1 || p->max_depth > 16) fail(GBDT_E_INVAL, "max_depth must be in [1, 16]");
    if (p->n_trees < 1) fail(GBDT_E_INVAL, "n_trees must be >= 1");
    if (!(p->lambda >= 0) || !std::isfinite(p->lambda)) fail(GBDT_E_INVAL, "lambda must be finite and >= 0");
    if (!(p->gamma >= 0) || !std::isfinite(p->gamma)) fail(GBDT_E_INVAL, "gamma must be finite and >= 0");
    if (!(p->eta > 0 && p->eta <= 1)) fail(GBDT_E_INVAL, "eta must be in (0, 1]");
    if (!std::isfinite(p->base_margin)) fail(GBDT_E_INVAL, "base_margin must be finite");
    if (p->loss != GBDT_LOSS_SQUARED && p->loss != GBDT_LOSS_LOGISTIC && p->loss != GBDT_LOSS_CUSTOM)
      fail(GBDT_E_INVAL, "unknown loss");
    if (p->loss == GBDT_LOSS_CUSTOM && !p->grad_fn) fail(GBDT_E_INVAL, "GBDT_LOSS_CUSTOM needs grad_fn");
    if (p->smartgd_off && !ds.rows_ptr.p) fail(GBDT_E_STATE, "smartgd_off needs a dataset loaded with keep_rows = 1");
    if (p->loss == GBDT_LOSS_LOGISTIC && (ds.h_labels_minmax[0] < 0 || ds.h_labels_minmax[1] > 1))
      fail(GBDT_E_INVAL, "logistic loss needs labels in [0, 1]");
    if (p->lambda == 0 && p->loss == GBDT_LOSS_LOGISTIC) {
      // H >= 1e-16 * count > 0, so every denominator of Eq. 2 stays positive: allowed
    }
    auto* m = new gbdt_model();
    try {
      train(ds, *p, m->m, train_margin);
    } catch (...) {
      delete m;
      throw;
    }
    *out = m;
  });
}

gbdt_status gbdt_predict(const gbdt_model* mh, int64_t n_rows, int64_t n_cols, const int64_t* indptr,
                         const int32_t* indices, const float* values, int32_t output_margin, double* out) {
  return guarded([&] {
    if (!mh || !out) fail(GBDT_E_INVAL, "NULL argument");
    if (mh->m.n_trees < 1) fail(GBDT_E_STATE, "model has no trees");
    validate_csr(n_rows, n_cols, indptr, indices, values, false);
    predict(mh->m, n_rows, n_cols, indptr, indices, values, output_margin, out, nullptr);
  });
}

gbdt_status gbdt_predict_on_stream(const gbdt_model* mh, int64_t n_rows, int64_t n_cols, const int64_t* indptr,
                                   const int32_t* indices, const float* values, int32_t output_margin, double* out,
                                   void* stream) {
  return guarded([&] {
    if (!mh || !out) fail(GBDT_E_INVAL, "NULL argument");
    if (mh->m.n_trees < 1) fail(GBDT_E_STATE, "model has no trees");
    validate_csr(n_rows, n_cols, indptr, indices, values, false);
    predict(mh->m, n_rows, n_cols, indptr, indices, values, output_margin, out, (cudaStream_t)stream);
  });
}

gbdt_status gbdt_model_export_level(const gbdt_model* mh, int32_t i, int64_t info[5], int64_t* col_start,
                                    int64_t* col_len, int64_t* seg_start, int64_t* seg_cnt, float* val, int32_t* ins,
                                    float* run_val, int32_t* run_len, int64_t* run_pos, int32_t* seg_run) {
  return guarded([&] {
    if (!mh || !info) fail(GBDT_E_INVAL, "NULL argument");
    const auto& caps = mh->m.captures;
    if (i < 0 || i >= (int32_t)caps.size()) fail(GBDT_E_STATE, "no captured level (set GBDT_CAPTURE_LEVEL before gbdt_train)");
    const LevelCapture& L = caps[i];
    info[0] = L.shard;
    info[1] = (int64_t)L.col_len.size();
    info[2] = L.K;
    info[3] = (int64_t)L.val.size();
    info[4] = (int64_t)L.run_val.size();
    auto cp = [](auto* dst, const auto& v) { if (dst) std::copy(v.begin(), v.end(), dst); };
    cp(col_start, L.col_start); cp(col_len, L.col_len); cp(seg_start, L.seg_start); cp(seg_cnt, L.seg_cnt);
    cp(val, L.val); cp(ins, L.ins); cp(run_val, L.run_val); cp(run_len, L.run_len); cp(run_pos, L.run_pos);
    cp(seg_run, L.seg_run);
  });
}

gbdt_status gbdt_model_train_loss(const gbdt_model* m, double* out) {
  return guarded([&] {
    if (!m || !out) fail(GBDT_E_INVAL, "NULL argument");
    for (size_t i = 0; i < m->m.train_loss.size(); ++i) out[i] = m->m.train_loss[i];
  });
}

gbdt_status gbdt_model_num_trees(const gbdt_model* m, int32_t* out) {
  return guarded([&] {
    if (!m || !out) fail(GBDT_E_INVAL, "NULL argument");
    *out = m->m.n_trees;
  });
}

gbdt_status gbdt_model_num_nodes(const gbdt_model* m, int32_t tree, int32_t* out) {
  return guarded([&] {
    if (!m || !out) fail(GBDT_E_INVAL, "NULL argument");
    if (tree < 0 || tree >= m->m.n_trees) fail(GBDT_E_RANGE, "tree index out of range");
    *out = (int32_t)m->m.nh();
  });
}

gbdt_status gbdt_model_export(const gbdt_model* m, int32_t tree, gbdt_node* nodes) {
  return guarded([&] {
    if (!m || !nodes) fail(GBDT_E_INVAL, "NULL argument");
    if (tree < 0 || tree >= m->m.n_trees) fail(GBDT_E_RANGE, "tree index out of range");
    const int64_t NH = m->m.nh();
    std::memcpy(nodes, m->m.nodes.data() + (size_t)tree * NH, sizeof(gbdt_node) * (size_t)NH);
  });
}

gbdt_status gbdt_get_timings(const gbdt_model* m, double* ms, int32_t n) {
  return guarded([&] {
    if (!m || !ms) fail(GBDT_E_INVAL, "NULL argument");
    for (int i = 0; i < n && i < GBDT_N_PHASES; ++i) ms[i] = m->m.timings[i];
  });
}

gbdt_status gbdt_get_level_entries(const gbdt_model* m, int64_t* entries, int32_t n) {
  return guarded([&] {
    if (!m || !entries) fail(GBDT_E_INVAL, "NULL argument");
    for (int i = 0; i < n; ++i) entries[i] = i < (int)m->m.level_entries.size() ? m->m.level_entries[i] : 0;
  });
}

gbdt_status gbdt_dataset_info(const gbdt_dataset* d, int32_t shard, int64_t info[7]) {
  return guarded([&] {
    if (!d || !info) fail(GBDT_E_INVAL, "NULL argument");
    const Dataset& ds = d->ds;
    if (shard < 0 || shard >= (int)ds.shards.size()) fail(GBDT_E_RANGE, "shard out of range");
    const Shard& s = *ds.shards[shard];
    info[0] = ds.n; info[1] = ds.m; info[2] = s.nnz; info[3] = (int64_t)ds.shards.size();
    info[4] = s.a_begin; info[5] = s.a_end; info[6] = s.rle ? s.runs : -1;
  });
}

gbdt_status gbdt_dataset_export_layout(const gbdt_dataset* d, int32_t shard, int64_t* col_ptr, float* val,
                                       int32_t* ins) {
  return guarded([&] {
    if (!d) fail(GBDT_E_INVAL, "NULL argument");
    const Dataset& ds = d->ds;
    if (shard < 0 || shard >= (int)ds.shards.size()) fail(GBDT_E_RANGE, "shard out of range");
    const Shard& s = *ds.shards[shard];
    GBDT_CUDA(cudaSetDevice(ds.device));
    int64_t off = 0;
    if (col_ptr) col_ptr[0] = 0;
    for (int a = 0; a < s.m; ++a) {
      const int64_t L = s.h_col_len[a];
      if (val && L) GBDT_CUDA(cudaMemcpy(val + off, s.val0.as<float>() + s.h_col_start[a], L * 4, cudaMemcpyDeviceToHost));
      if (ins && L) GBDT_CUDA(cudaMemcpy(ins + off, s.ins0.as<int32_t>() + s.h_col_start[a], L * 4, cudaMemcpyDeviceToHost));
      off += L;
      if (col_ptr) col_ptr[a + 1] = off;
    }
  });
}

gbdt_status gbdt_dataset_export_rle(const gbdt_dataset* d, int32_t shard, int64_t* run_ptr, float* run_val,
                                    int32_t* run_len) {
  return guarded([&] {
    if (!d) fail(GBDT_E_INVAL, "NULL argument");
    const Dataset& ds = d->ds;
    if (shard < 0 || shard >= (int)ds.shards.size()) fail(GBDT_E_RANGE, "shard out of range");
    const Shard& s = *ds.shards[shard];
    if (!s.rle) fail(GBDT_E_STATE, "shard is not RLE-compressed");
    GBDT_CUDA(cudaSetDevice(ds.device));
    if (run_ptr) GBDT_CUDA(cudaMemcpy(run_ptr, s.run_ptr.p, (size_t)(s.m + 1) * 8, cudaMemcpyDeviceToHost));
    if (run_val && s.runs) GBDT_CUDA(cudaMemcpy(run_val, s.run_val.p, (size_t)s.runs * 4, cudaMemcpyDeviceToHost));
    if (run_len && s.runs) GBDT_CUDA(cudaMemcpy(run_len, s.run_len.p, (size_t)s.runs * 4, cudaMemcpyDeviceToHost));
  });
}

gbdt_status gbdt_shard_ranges(int64_t n_cols, const int64_t* col_counts, int32_t P, int32_t* bounds) {
  return guarded([&] {
    if ((!col_counts && n_cols > 0) || !bounds) fail(GBDT_E_INVAL, "NULL argument");
    if (n_cols < 0 || n_cols >= (int64_t(1) << 31)) fail(GBDT_E_INVAL, "n_cols out of range");
    if (P < 1 || P > 8 || (P & (P - 1))) fail(GBDT_E_RANGE, "P must be 1, 2, 4 or 8");
    for (int64_t a = 0; a < n_cols; ++a)
      if (col_counts[a] < 0) fail(GBDT_E_INVAL, "negative column count");
    const std::vector<int32_t> b = shard_ranges(n_cols, col_counts, P);
    std::copy(b.begin(), b.end(), bounds);
  });
}

gbdt_status gbdt_comm_init_callbacks(int32_t rank, int32_t world, gbdt_allgather_fn allgather,
                                     gbdt_allreduce_u8_fn allreduce_u8, void* user, int32_t device,
                                     gbdt_comm** out) {
  if (out) *out = nullptr;
  return guarded([&] {
    if (!allgather || !allreduce_u8 || !out) fail(GBDT_E_INVAL, "NULL argument");
    if (world < 1 || world > 8 || (world & (world - 1))) fail(GBDT_E_RANGE, "world must be 1, 2, 4 or 8");
    if (rank < 0 || rank >= world) fail(GBDT_E_RANGE, "rank out of range");
    if (device >= 0) GBDT_CUDA(cudaSetDevice(device));
    int dev = 0;
    GBDT_CUDA(cudaGetDevice(&dev));
    auto* c = new gbdt_comm();
    c->c = new Comm();
    c->c->rank = rank;
    c->c->world = world;
    c->c->device = dev;
    c->c->cb_allgather = allgather;
    c->c->cb_allreduce = allreduce_u8;
    c->c->cb_user = user;
    *out = c;
  });
}

gbdt_status gbdt_comm_unique_id(uint8_t id[128]) {
  return guarded([&] {
    if (!id) fail(GBDT_E_INVAL, "NULL argument");
    comm_unique_id(id);
  });
}

gbdt_status gbdt_comm_init(int32_t rank, int32_t world, const uint8_t id[128], int32_t device, gbdt_comm** out) {
  if (out) *out = nullptr;
  return guarded([&] {
    if (!id || !out) fail(GBDT_E_INVAL, "NULL argument");
    if (world < 1 || world > 8 || (world & (world - 1))) fail(GBDT_E_RANGE, "world must be 1, 2, 4 or 8");
    if (rank < 0 || rank >= world) fail(GBDT_E_RANGE, "rank out of range");
    auto* c = new gbdt_comm();
    c->c = comm_init(rank, world, id, device);
    *out = c;
  });
}

void gbdt_comm_free(gbdt_comm* c) {
  if (!c) return;
  comm_free(c->c);
  delete c;
}

void gbdt_dataset_free(gbdt_dataset* d) {
  if (!d) return;
  cudaSetDevice(d->ds.device);
  cudaStream_t st = d->ds.stream;
  delete d;
  cudaStreamSynchronize(st);
}

void gbdt_model_free(gbdt_model* m) { delete m; }

}  // extern "C"
