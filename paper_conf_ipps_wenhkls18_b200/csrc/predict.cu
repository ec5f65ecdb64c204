// predict.cu -- GPU-GBDT prediction: the trees are applied in order to every row;
// a row goes high/left iff its value of the split attribute is >= split_value, missing values
// follow the stored default direction (reading R11 of the garbled P:279).
//
// One thread per row walks all trees in order and accumulates yhat = base + sum_t eta * w_t with
// the same explicitly rounded ops as the training-time SmartGD update, so that predicting the
// training rows reproduces the cached training margin bit for bit.  Rows of at most 64 columns
// are looked up in a dense shared-memory table; wider rows by binary search in the CSR row.
#include <algorithm>

#include "common.cuh"

namespace gbdt {
namespace {

__global__ void k_predict(int64_t n, const int64_t* __restrict__ indptr, const int32_t* __restrict__ indices,
                          const float* __restrict__ values, const gbdt_node* __restrict__ nodes, int n_trees,
                          int64_t NH, double eta, double base, int sigmoid, double* __restrict__ out) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    double y = base;
    for (int t = 0; t < n_trees; ++t) {
      y = __dadd_rn(y, __dmul_rn(eta, tree_leaf_weight(nodes + (int64_t)t * NH, indptr, indices, values, i)));
    }
    if (sigmoid) y = __ddiv_rn(1.0, __dadd_rn(1.0, exp(-y)));
    out[i] = y;
  }
}

// Rows with few columns (n_cols <= kDenseCols): a block's 128 rows are staged as a dense table in
// shared memory (NaN = missing), filled cooperatively by coalesced loads of the block's contiguous
// CSR range, so every node visit is one shared-memory read instead of a binary search.
constexpr int kDenseCols = 64;
constexpr int kPredRows = 128;
__global__ void __launch_bounds__(kPredRows) k_predict_dense(int64_t n, int m, const int64_t* __restrict__ indptr,
                                                             const int32_t* __restrict__ indices,
                                                             const float* __restrict__ values,
                                                             const gbdt_node* __restrict__ nodes, int n_trees,
                                                             int64_t NH, double eta, double base, int sigmoid,
                                                             double* __restrict__ out) {
  __shared__ float X[kPredRows][kDenseCols + 1];
  __shared__ int64_t rp[kPredRows + 1];
  const int tid = threadIdx.x;
  for (int64_t r0 = (int64_t)blockIdx.x * kPredRows; r0 < n; r0 += (int64_t)gridDim.x * kPredRows) {
    const int rows = (int)min((int64_t)kPredRows, n - r0);
    for (int a = 0; a < kDenseCols; ++a) X[tid][a] = __int_as_float(0x7fc00000);  // missing
    for (int q = tid; q <= rows; q += kPredRows) rp[q] = indptr[r0 + q];
    __syncthreads();
    const int64_t e0 = rp[0], e1 = rp[rows];
    for (int64_t e = e0 + tid; e < e1; e += kPredRows) {
      int lo = 0, hi = rows - 1;  // the row holding entry e: largest q with rp[q] <= e
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (rp[mid] <= e) lo = mid; else hi = mid - 1;
      }
      const int a = indices[e];
      if (a < m) {
        const float v = values[e];
        X[lo][a] = v == 0.0f ? 0.0f : v;  // -0.0 reads as +0.0, NaN stays missing
      }
    }
    __syncthreads();
    if (tid < rows) {
      double y = base;
      for (int t = 0; t < n_trees; ++t) {
        const gbdt_node* T = nodes + (int64_t)t * NH;
        int64_t k = 0;
        while (!T[k].is_leaf) {
          const float x = X[tid][T[k].attr];
          const bool high = isnan(x) ? (T[k].default_left != 0) : (x >= T[k].split_value);
          k = high ? 2 * k + 1 : 2 * k + 2;
        }
        y = __dadd_rn(y, __dmul_rn(eta, T[k].weight));
      }
      if (sigmoid) y = __ddiv_rn(1.0, __dadd_rn(1.0, exp(-y)));
      out[r0 + tid] = y;
    }
    __syncthreads();
  }
}

}  // namespace

void predict(const Model& m, int64_t n_rows, int64_t n_cols, const int64_t* indptr, const int32_t* indices,
             const float* values, int output_margin, double* out, cudaStream_t st) {
  GBDT_CUDA(cudaSetDevice(m.device));
  const int64_t nnz = indptr[n_rows];
  const int64_t NH = m.nh();
  DBuf dptr((size_t)(n_rows + 1) * 8, st), didx((size_t)std::max<int64_t>(nnz, 1) * 4, st),
      dval((size_t)std::max<int64_t>(nnz, 1) * 4, st), dnodes(m.nodes.size() * sizeof(gbdt_node), st),
      dout((size_t)std::max<int64_t>(n_rows, 1) * 8, st);
  GBDT_CUDA(cudaMemcpyAsync(dptr.p, indptr, (size_t)(n_rows + 1) * 8, cudaMemcpyHostToDevice, st));
  if (nnz) {
    GBDT_CUDA(cudaMemcpyAsync(didx.p, indices, (size_t)nnz * 4, cudaMemcpyHostToDevice, st));
    GBDT_CUDA(cudaMemcpyAsync(dval.p, values, (size_t)nnz * 4, cudaMemcpyHostToDevice, st));
  }
  if (m.dense) {  // trained on the dense representation: absent values are filled here too
    DBuf fptr, fidx, fval;
    densify(n_rows, m.n_cols, dptr.as<int64_t>(), didx.as<int32_t>(), dval.as<float>(), m.fill, fptr, fidx, fval, st);
    dptr = std::move(fptr);
    didx = std::move(fidx);
    dval = std::move(fval);
  }
  GBDT_CUDA(cudaMemcpyAsync(dnodes.p, m.nodes.data(), m.nodes.size() * sizeof(gbdt_node), cudaMemcpyHostToDevice, st));
  const int sig = (!output_margin && m.loss == GBDT_LOSS_LOGISTIC) ? 1 : 0;
  if (m.n_cols <= kDenseCols) {  // split attributes are < the training n_cols; other columns are ignored
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n_rows, kPredRows), 148 * 16));
    k_predict_dense<<<grid, kPredRows, 0, st>>>(n_rows, (int)m.n_cols, dptr.as<int64_t>(), didx.as<int32_t>(),
                                                dval.as<float>(), dnodes.as<gbdt_node>(), m.n_trees, NH, m.eta,
                                                m.base_margin, sig, dout.as<double>());
  } else {
    const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n_rows, 256), 148 * 16));
    k_predict<<<grid, 256, 0, st>>>(n_rows, dptr.as<int64_t>(), didx.as<int32_t>(), dval.as<float>(),
                                    dnodes.as<gbdt_node>(), m.n_trees, NH, m.eta, m.base_margin, sig,
                                    dout.as<double>());
  }
  GBDT_LAUNCH_CHECK();
  count_launch();
  GBDT_CUDA(cudaMemcpyAsync(out, dout.p, (size_t)n_rows * 8, cudaMemcpyDeviceToHost, st));
  GBDT_CUDA(cudaStreamSynchronize(st));
  (void)n_cols;
}

}  // namespace gbdt
