// predict.cu -- GPU-GBDT prediction: the trees are applied in order to every row;
// a row goes high/left iff its value of the split attribute is >= split_value, missing values
// follow the stored default direction (reading R11 of the garbled P:279).
//
// One thread per row walks all trees in order and accumulates yhat = base + sum_t eta * w_t with
// the same explicitly rounded ops as the training-time SmartGD update, so that predicting the
// training rows reproduces the cached training margin bit for bit.
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

}  // namespace

void predict(const Model& m, int64_t n_rows, int64_t n_cols, const int64_t* indptr, const int32_t* indices,
             const float* values, int output_margin, double* out) {
  GBDT_CUDA(cudaSetDevice(m.device));
  cudaStream_t st = nullptr;
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
  GBDT_CUDA(cudaMemcpyAsync(dnodes.p, m.nodes.data(), m.nodes.size() * sizeof(gbdt_node), cudaMemcpyHostToDevice, st));
  const int sig = (!output_margin && m.loss == GBDT_LOSS_LOGISTIC) ? 1 : 0;
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n_rows, 256), 148 * 16));
  k_predict<<<grid, 256, 0, st>>>(n_rows, dptr.as<int64_t>(), didx.as<int32_t>(), dval.as<float>(),
                                  dnodes.as<gbdt_node>(), m.n_trees, NH, m.eta, m.base_margin, sig,
                                  dout.as<double>());
  GBDT_LAUNCH_CHECK();
  count_launch();
  GBDT_CUDA(cudaMemcpyAsync(out, dout.p, (size_t)n_rows * 8, cudaMemcpyDeviceToHost, st));
  GBDT_CUDA(cudaStreamSynchronize(st));
  (void)n_cols;
}

}  // namespace gbdt
