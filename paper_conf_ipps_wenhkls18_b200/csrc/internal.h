// internal.h -- host-side structures of libgbdt.so (not part of the C ABI).
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <memory>
#include <string>
#include <vector>

#include "../../include/gbdt.h"

namespace gbdt {

constexpr int kMaxDevices = 64;  // device ordinals the library keeps per-device state for

struct Error {
  gbdt_status st;
  std::string msg;
};

[[noreturn]] void fail(gbdt_status st, const std::string& msg);

#define GBDT_CUDA(x)                                                                        \
  do {                                                                                      \
    cudaError_t e_ = (x);                                                                   \
    if (e_ != cudaSuccess)                                                                  \
      ::gbdt::fail(e_ == cudaErrorMemoryAllocation ? GBDT_E_NOMEM : GBDT_E_CUDA,            \
                   std::string(#x) + ": " + cudaGetErrorString(e_) + " (" __FILE__ ":" +    \
                       std::to_string(__LINE__) + ")");                                     \
  } while (0)

#define GBDT_LAUNCH_CHECK() GBDT_CUDA(cudaGetLastError())

// Counts kernel launches of the current gbdt_train (bench "gpu_launches" evidence).
void count_launch(int k = 1);

// Stream-ordered device buffer (cudaMallocAsync / cudaFreeAsync).
struct DBuf {
  void* p = nullptr;
  size_t bytes = 0;
  cudaStream_t st = nullptr;
  DBuf() = default;
  DBuf(size_t b, cudaStream_t s) { alloc(b, s); }
  void alloc(size_t b, cudaStream_t s);
  void release();
  ~DBuf() { release(); }
  DBuf(const DBuf&) = delete;
  DBuf& operator=(const DBuf&) = delete;
  DBuf(DBuf&& o) noexcept { *this = std::move(o); }
  DBuf& operator=(DBuf&& o) noexcept {
    if (this != &o) {
      release();
      p = o.p; bytes = o.bytes; st = o.st;
      o.p = nullptr; o.bytes = 0;
    }
    return *this;
  }
  template <class T> T* as() const { return static_cast<T*>(p); }
};

// Per-level attribute/segment tables of one shard (device pointers).
// Segment s = a*K + j is node j's part of attribute a's list; it occupies
// [seg_start[s], seg_start[s] + seg_cnt[s]) of the level buffer.
struct Tables {
  int64_t* col_start = nullptr;   // [m+1] padded start of each attribute list
  int64_t* col_len = nullptr;     // [m]   entries of each attribute list at this level
  int32_t* tile_start = nullptr;  // [m+1] first tile of each attribute (tiles never straddle)
  int32_t* chunk_start = nullptr; // [m+1] first 256-entry chunk of each attribute (8 per tile)
  int64_t* seg_start = nullptr;   // [m*Kcap]
  int64_t* seg_cnt = nullptr;     // [m*Kcap]
  int32_t* T = nullptr;           // [1] tiles at this level
  int32_t* C = nullptr;           // [1] chunks at this level
  int32_t* chunk_attr = nullptr;  // [C] attribute of each chunk
  // RLE: the runs of segment s are [seg_run[s], seg_run[s+1]); run r covers list
  // positions [run_pos[r], run_pos[r] + run_len[r]) with value run_val[r]
  int32_t* seg_run = nullptr;     // [m*Kcap + 1]
  float* run_val = nullptr;
  int32_t* run_len = nullptr;
  int64_t* run_pos = nullptr;
  int32_t* R = nullptr;           // [1] runs at this level
  int32_t* run_chunk = nullptr;   // [C] the run holding each chunk's first entry
  // short-attribute path (levels.cu k_short_*): the chunks the chunk kernels take, i.e. those of
  // the attributes not on the short path (all chunks when nullptr, or when K > 32)
  int32_t* lc = nullptr;          // [C]
  int32_t* nlc = nullptr;         // [1]
};

// Best split of one node found in one shard ("piece" records are reduced to this).
struct Rec {
  double gain;
  double GL, HL;      // high/left child totals (include the missing part when dir == 1)
  long long cntL;     // high/left child instance count
  long long pos;      // level-buffer position of the last present high entry (owner shard)
  float value;        // split value (smallest value on the high side)
  int attr;           // global attribute id
  int dir;            // 1: missing -> high/left
  int node;           // node index at this level
  int epoch;          // level epoch that produced it
  int shard;          // owner shard (global index)
};

struct Comm;  // comm.cpp

struct Shard {
  int32_t index = 0;             // global shard index
  int32_t a_begin = 0, a_end = 0, m = 0;
  int64_t nnz = 0;               // stored entries of this shard
  int64_t cap = 0;               // padded level-buffer length (+ slack)
  int32_t T0 = 0;                // tiles at the root
  int32_t C0 = 0;                // 256-entry chunks at the root
  DBuf val0, ins0;               // pristine root layout (padded)
  DBuf valw[2], insw[2];         // ping-pong level buffers
  DBuf root_tab;                 // root tables storage
  DBuf root_chunk_attr;
  Tables root;
  std::vector<int64_t> h_col_len;  // host copy, unpadded lengths
  std::vector<int64_t> h_col_start;
  // RLE
  bool rle = false;
  int64_t runs = 0;
  DBuf run_ptr, run_val, run_len, run_pos, run_seg, run_chunk;
};

struct Dataset {
  int64_t n = 0, m = 0, nnz = 0;
  int device = 0;
  cudaStream_t stream = nullptr;
  bool has_missing = false;      // some instance lacks some attribute
  bool binary_labels = false;    // every label is 0 or 1
  DBuf y;                        // labels (device, fp32)
  std::vector<float> h_labels_minmax;  // [min, max]
  std::vector<std::unique_ptr<Shard>> shards;  // local shards
  int32_t n_total_shards = 1;    // across all ranks
  Comm* comm = nullptr;
  int rle = 0;
  int dense = 0;                 // dense representation: absent values were filled
  float fill = 0.f;
  DBuf rows_ptr, rows_idx, rows_val;  // CSR rows (gbdt_load_opts.keep_rows; SmartGD-off ablation)
};

// One shard's level lists and tables (test hook GBDT_CAPTURE_LEVEL; gbdt_model_export_level)
struct LevelCapture {
  int shard = 0, K = 0;
  std::vector<int64_t> col_start, col_len, seg_start, seg_cnt, run_pos;
  std::vector<float> val, run_val;
  std::vector<int32_t> ins, run_len, seg_run;
};

struct Model {
  int32_t n_trees = 0, max_depth = 0, loss = 0;
  int64_t n_cols = 0;
  double eta = 0, base_margin = 0, lambda = 0;
  std::vector<gbdt_node> nodes;  // n_trees * NH
  double timings[GBDT_N_PHASES] = {0};
  std::vector<int64_t> level_entries;  // [max_depth] list entries scanned per level (profile = 1)
  std::vector<double> train_loss;      // [n_trees + 1] mean training loss after 0 .. T trees
  std::vector<LevelCapture> captures;  // per local shard (GBDT_CAPTURE_LEVEL)
  int device = 0;
  int dense = 0;                 // trained on the dense representation: predict fills absent values
  float fill = 0.f;
  int64_t nh() const { return (int64_t(1) << (max_depth + 1)) - 1; }
};

struct Comm {
  int rank = 0, world = 1, device = 0;
  void* nccl = nullptr;  // ncclComm_t
  // host-staged callback collectives (gbdt_comm_init_callbacks); used when nccl == nullptr
  gbdt_allgather_fn cb_allgather = nullptr;
  gbdt_allreduce_u8_fn cb_allreduce = nullptr;
  void* cb_user = nullptr;
  void allgather(const void* send, void* recv, size_t bytes, cudaStream_t st);
  void allreduce_sum_u8(void* buf, size_t n, cudaStream_t st);
};

// api.cpp: contiguous attribute ranges balanced by entries
std::vector<int32_t> shard_ranges(int64_t n_cols, const int64_t* col_counts, int P);
// layout.cu
std::vector<int64_t> column_counts(int64_t nnz, int64_t m, const int32_t* d_indices, const float* d_values,
                                   cudaStream_t st);
void build_layout(Dataset& ds, const int64_t* d_indptr, const int32_t* d_indices,
                  const float* d_values, const std::vector<int64_t>& col_counts,
                  double rle_min_ratio);
std::vector<uint32_t> attribute_runs(const Shard& sh, cudaStream_t st, int sms);
void densify(int64_t n, int64_t m, const int64_t* d_indptr, const int32_t* d_idx, const float* d_val, float fill,
             DBuf& optr, DBuf& oidx, DBuf& oval, cudaStream_t st);
// train.cu
void train(Dataset& ds, const gbdt_params& p, Model& model, double* margin_out);
// predict.cu
void predict(const Model& m, int64_t n_rows, int64_t n_cols, const int64_t* indptr,
             const int32_t* indices, const float* values, int output_margin, double* out, cudaStream_t st);

inline int64_t pad4(int64_t x) { return (x + 3) & ~int64_t(3); }
inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

}  // namespace gbdt
