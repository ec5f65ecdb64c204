/*
 * gbdt.h -- C ABI of the B200-native exact-greedy GBDT hot path (libgbdt.so).
 *
 * Method: Wen, He, Ramamohanarao, Lu, Shi, "Efficient Gradient Boosted Decision Tree Training on
 * GPUs", IPDPS 2018 (text in /root/reference/PAPER.md; "P:<n>" = line n of that file).
 *
 *   Training (Alg. 1): trees are built one after another; every tree is grown level
 *   by level over attribute-major lists sorted by value, optionally run-length
 *   encoded.  Per level: segmented prefix sum of (g, h) over the (node, attribute)
 *   segments, gain of every distinct split value (Eq. 2; repeated values and
 *   runs skipped; missing values tried on both sides), best split
 *   per node and split iff gain > gamma, then an order-preserving partition
 *   of every segment into its two children (RLE runs split without decompression,
 *   P:250).  Gradients come from the cached prediction updated with the previous tree's leaf
 *   weights ("SmartGD").
 *
 * Conventions shared by every entry point
 *   - extern "C", C11 types only; no exception crosses the ABI.
 *   - Every function returns a gbdt_status; on failure the thread-local message is available
 *     through gbdt_last_error(), output handles are set to NULL and caller buffers are untouched.
 *   - Host pointers are caller-owned, read only during the call and copied.  Handles are
 *     library-owned until the matching *_free.  A handle must not be used by two threads at once.
 *   - Values: NaN = missing; -0.0 is treated as +0.0; +-Inf are ordinary values.
 *   - Precision: attribute values fp32; g, h, predictions, all sums, gains, weights fp64.
 *   - There is no CPU fallback: without a usable CUDA device every call returns GBDT_E_CUDA.
 */
#ifndef GBDT_H_
#define GBDT_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct gbdt_dataset gbdt_dataset; /* opaque: device-resident attribute-major layout */
typedef struct gbdt_model gbdt_model;     /* opaque: host-resident trees (+ device copy) */
typedef struct gbdt_comm gbdt_comm;       /* opaque: NCCL communicator for attribute sharding */

typedef enum {
  GBDT_OK = 0,
  GBDT_E_INVAL = 1,  /* malformed argument (CSR structure, labels, parameters) */
  GBDT_E_NOMEM = 2,  /* device or host allocation failed */
  GBDT_E_CUDA = 3,   /* CUDA runtime/driver error, or no device */
  GBDT_E_NCCL = 4,   /* NCCL error or NCCL library not loadable */
  GBDT_E_STATE = 5,  /* handle in the wrong state (e.g. predict on an empty model) */
  GBDT_E_RANGE = 6   /* a count outside the supported range (shards, devices, sizes) */
} gbdt_status;

typedef enum { GBDT_LOSS_SQUARED = 0, GBDT_LOSS_LOGISTIC = 1, GBDT_LOSS_CUSTOM = 2 } gbdt_loss;

/* User-defined loss (GBDT_LOSS_CUSTOM; the paper's "users can define their own loss function",
 * P:193).  Called once per tree, after the cached prediction has been updated
 * (SmartGD), with DEVICE pointers: yhat, labels (n each, read only) and g, h (n each, to be
 * written: first and second derivative of the loss at yhat, h >= 0 and finite).  The callback
 * must enqueue its work on `stream` (the library's cudaStream_t) or complete it before
 * returning; the library reads g and h in stream order afterwards.  Returns 0 on success; any
 * other value aborts the gbdt_train with GBDT_E_INVAL.  `user` is gbdt_params.grad_user. */
typedef int (*gbdt_grad_fn)(int64_t n, const double* yhat, const float* labels, double* g, double* h,
                            void* stream, void* user);
typedef enum { GBDT_RLE_OFF = 0, GBDT_RLE_ON = 1, GBDT_RLE_AUTO = 2 } gbdt_rle;

/* Options of gbdt_load_csr.  Zero-initialised means: no RLE, one shard, current device,
 * default stream, no communicator. */
typedef struct {
  int32_t rle;            /* gbdt_rle.  RLE of the sorted lists.  AUTO compresses an
                             attribute when entries/runs >= rle_min_ratio (reading R21 of the
                             paper's "dimensionality/cardinality > R"). */
  double rle_min_ratio;   /* AUTO threshold; <= 0 means 2.0 */
  int32_t n_shards;       /* attribute shards held by THIS process on its device (loopback
                             sharding; 0 or 1 = unsharded).  1, 2, 4 or 8.  Used to test the
                             multi-GPU merge on one device: trees are bit-identical for any k. */
  int32_t device;         /* CUDA device ordinal; < 0 = the current device */
  void* stream;           /* cudaStream_t for every launch and copy; NULL = legacy default */
  gbdt_comm* comm;        /* NULL: single process.  Else this process is rank r of a world of
                             size w and owns attribute range r of w (nnz-balanced, contiguous);
                             n_shards must then be 0 or 1. */
  int32_t keep_rows;      /* 1: keep a device copy of the CSR rows (needed by smartgd_off) */
  int32_t dense;          /* 1: dense representation (the paper's option "if the data set is
                             small"): the n_rows x n_cols matrix with every absent or
                             NaN value replaced by dense_fill ("in the dense presentation, missing
                             values need to be filled (e.g., treated as 0)").  The trees then
                             see no missing values; models trained this way fill absent values at
                             predict time too.  Memory: n_rows * n_cols entries. */
  float dense_fill;       /* the fill value (0 when zero-initialised) */
} gbdt_load_opts;

/* Training parameters, as the paper states them: d, T, gamma (Alg. 1 inputs),
 * lambda (Eq. 2), eta (learning rate), loss. */
typedef struct {
  int32_t max_depth;      /* d in [1, 16]; root has depth 0, nodes with depth < d may split */
  int32_t n_trees;        /* T >= 1 */
  double lambda;          /* >= 0 */
  double gamma;           /* >= 0; a node splits iff best gain > max(gamma, 0) */
  double eta;             /* (0, 1]; yhat += eta * w_leaf */
  double base_margin;     /* initial prediction (reading R7) */
  int32_t loss;           /* gbdt_loss */
  int32_t profile;        /* 1: record per-phase device times (gbdt_get_timings) */
  int32_t smartgd_off;    /* 1: ablation of SmartGD (Fig. 9): before every tree each
                             instance's prediction is recomputed by traversing all previous trees
                             over its CSR row instead of adding its last leaf weight.  Same
                             arithmetic in the same order, so the trees are bit-identical.  Needs
                             a dataset loaded with keep_rows = 1 (else GBDT_E_STATE). */
  int32_t rle_decompress; /* RLE shards only: 0 = split the runs directly (Fig. 7); 1 = the
                             paper's baseline "splitting RLE with decompression" (Fig. 6):
                             decompress, partition the plain lists, re-encode the children.  The
                             trees are identical; this is the ablation of P:536. */
  gbdt_grad_fn grad_fn;   /* GBDT_LOSS_CUSTOM: the gradient callback (else ignored) */
  void* grad_user;        /* passed through to grad_fn */
} gbdt_params;

/* One tree node in heap order: root 0, children of k are 2k+1 (high/left: x >= split_value)
 * and 2k+2 (low/right).  Unused heap slots have heap_id == -1. */
typedef struct {
  int32_t heap_id;
  int32_t is_leaf;
  int32_t attr;          /* split attribute (global column id); -1 for leaves */
  int32_t default_left;  /* 1: missing values go to the high/left child */
  float split_value;     /* smallest value on the high side (a data value, reading R11) */
  int32_t reserved;
  double gain;           /* Eq. 2 gain of the split (0 for leaves) */
  double G, H;           /* sums of g and h over the node's instances */
  double weight;         /* leaf weight -G/(H+lambda) (reading R3); 0 for internal nodes */
  int64_t count;         /* instances in the node */
} gbdt_node;

/* Phases reported by gbdt_get_timings (milliseconds of device time, summed over the run). */
enum {
  GBDT_PHASE_GRAD = 0,       /* SmartGD gradients + root totals */
  GBDT_PHASE_SPLIT_FIND = 1, /* segmented scan + gain + per-piece argmax */
  GBDT_PHASE_DECIDE = 2,     /* per-node argmax merge, split decision, tree emission */
  GBDT_PHASE_NODEMAP = 3,    /* instance -> child bitmap and node map */
  GBDT_PHASE_PARTITION = 4,  /* order-preserving partition */
  GBDT_PHASE_COMM = 5,       /* NCCL allgather of node bests + bitmap allreduce */
  GBDT_PHASE_TOTAL = 6,      /* whole gbdt_train on the device */
  /* kernel-level timers nested inside the phases above (profile = 1): */
  GBDT_PHASE_K_CHUNK_AGG = 7, /* k_chunk_agg + exact carry scan (inside SPLIT_FIND) */
  GBDT_PHASE_K_SPLIT = 8,     /* k_sf_fast + k_sf_gen: scan, gains, node bests (inside SPLIT_FIND) */
  GBDT_PHASE_K_COUNT = 9,     /* k_part_count + count scan + plan (inside PARTITION) */
  GBDT_PHASE_K_SCATTER = 10,  /* k_part_scatter (+ RLE run split) (inside PARTITION) */
  GBDT_PHASE_K_FUSED = 11,    /* dense data: k_fused, the partition of level l and the split find
                                 of level l+1 in one pass (inside PARTITION) */
  GBDT_N_PHASES = 12
};

/* Copies a CSR matrix (indptr int64[n_rows+1], indices int32[nnz] strictly increasing per row,
 * values float32[nnz]) and labels float32[n_rows] to the device and builds the attribute-major
 * layout: per attribute the present entries sorted by value descending, ties by ascending
 * instance id, optionally RLE-compressed.
 * Errors: GBDT_E_INVAL if n_rows or n_cols is outside [1, 2^31-1), indptr[0] != 0, indptr is
 * decreasing, an index is out of range or not strictly increasing within its row, nnz >= 2^31,
 * or a label is not finite; GBDT_E_RANGE for an unsupported n_shards; GBDT_E_CUDA / NOMEM. */
gbdt_status gbdt_load_csr(int64_t n_rows, int64_t n_cols, const int64_t* indptr,
                          const int32_t* indices, const float* values, const float* labels,
                          const gbdt_load_opts* opts, gbdt_dataset** out);

/* Trains p->n_trees trees on ds (Alg. 1).  Logistic loss needs labels in [0, 1].
 * train_margin: nullable host buffer of n_rows doubles, receives the final cached prediction
 * yhat (base_margin + eta * sum of leaf weights), identical to gbdt_predict on the training
 * rows.  The dataset stays loaded and can be trained again.
 * Errors: GBDT_E_INVAL for parameters outside the ranges documented in gbdt_params. */
gbdt_status gbdt_train(gbdt_dataset* ds, const gbdt_params* p, gbdt_model** out,
                       double* train_margin);

/* Predicts rows given as CSR (same conventions as gbdt_load_csr) with the model's trees in
 * order: out[i] = base_margin + sum_t eta * w_t(leaf_t(i)) (output_margin = 1) or
 * its sigmoid for logistic models (output_margin = 0).  A column id >= the training n_cols is
 * treated as missing.  out: caller-owned host buffer of n_rows doubles. */
gbdt_status gbdt_predict(const gbdt_model* m, int64_t n_rows, int64_t n_cols,
                         const int64_t* indptr, const int32_t* indices, const float* values,
                         int32_t output_margin, double* out);
/* gbdt_predict with every copy and launch on the caller's cudaStream_t `stream` (NULL = the legacy
 * default stream, which is what gbdt_predict uses).  Returns after the result is in `out`. */
gbdt_status gbdt_predict_on_stream(const gbdt_model* m, int64_t n_rows, int64_t n_cols,
                                   const int64_t* indptr, const int32_t* indices, const float* values,
                                   int32_t output_margin, double* out, void* stream);

/* Model inspection.  Nodes are returned in heap order, 2^(max_depth+1)-1 slots per tree. */
gbdt_status gbdt_model_num_trees(const gbdt_model* m, int32_t* out);
gbdt_status gbdt_model_num_nodes(const gbdt_model* m, int32_t tree, int32_t* out);
gbdt_status gbdt_model_export(const gbdt_model* m, int32_t tree, gbdt_node* nodes);

/* Mean training loss of the model after 0, 1, ..., n_trees trees (out: n_trees + 1 doubles,
 * caller-owned): squared (y - yhat)^2, logistic the cross-entropy of P:120; the paper's RMSE
 * (Table II) is the square root of the squared-loss entries.  NaN for a custom loss. */
gbdt_status gbdt_model_train_loss(const gbdt_model* m, double* out);

/* Test hook for the kernel-level invariants (every child segment equals the root
 * column filtered by node membership, Fig. 2; with RLE its runs equal RLE of that,
 * P:250 Fig. 7).  When the environment variable GBDT_CAPTURE_LEVEL=l is set at gbdt_train time
 * (level-by-level path, eager launches), the lists of level l of tree 0 are copied into the model,
 * one capture per local shard i.  info[5] = {shard, m_shard, K (nodes), list length (padded),
 * runs}; call with NULL arrays first to size them.  Arrays: col_start[m+1] (padded list starts),
 * col_len[m], seg_start[m*K], seg_cnt[m*K] (segment a*K+j = node j's part of attribute a),
 * val/ins[list length], RLE: run_val/run_len/run_pos[runs], seg_run[m*K+1].  Any may be NULL.
 * GBDT_E_STATE if nothing was captured. */
gbdt_status gbdt_model_export_level(const gbdt_model* m, int32_t shard, int64_t info[5], int64_t* col_start,
                                    int64_t* col_len, int64_t* seg_start, int64_t* seg_cnt, float* val,
                                    int32_t* ins, float* run_val, int32_t* run_len, int64_t* run_pos,
                                    int32_t* seg_run);

/* Per-phase device milliseconds of the gbdt_train that produced m (profile = 1), else zeros.
 * ms_by_phase: caller-owned, n_phases entries (<= GBDT_N_PHASES filled). */
gbdt_status gbdt_get_timings(const gbdt_model* m, double* ms_by_phase, int32_t n_phases);

/* Entries of the local shards' attribute lists that split finding scanned at each level, summed
 * over the trees of the gbdt_train that produced m (profile = 1; else zeros).  This is the unit of
 * the bench's byte model (bytes per entry x entries).  entries: caller-owned, n_levels entries
 * (level l < max_depth filled, the rest zeroed). */
gbdt_status gbdt_get_level_entries(const gbdt_model* m, int64_t* entries, int32_t n_levels);

/* Dataset inspection (tests): sizes and the built layout of one shard.
 * info: [n_rows, n_cols, nnz_stored, n_shards, attr_begin(shard), attr_end(shard), rle_runs(shard)]. */
gbdt_status gbdt_dataset_info(const gbdt_dataset* ds, int32_t shard, int64_t info[7]);
/* Copies shard's sorted lists to host: col_ptr int64[m_shard+1] (unpadded offsets), val
 * float32[nnz_shard], ins int32[nnz_shard].  Any pointer may be NULL. */
gbdt_status gbdt_dataset_export_layout(const gbdt_dataset* ds, int32_t shard, int64_t* col_ptr,
                                       float* val, int32_t* ins);
/* Copies shard's RLE runs (GBDT_RLE_ON/AUTO): run_ptr int64[m_shard+1], run_val float32[R],
 * run_len int32[R].  GBDT_E_STATE if the shard is not RLE-compressed. */
gbdt_status gbdt_dataset_export_rle(const gbdt_dataset* ds, int32_t shard, int64_t* run_ptr,
                                    float* run_val, int32_t* run_len);

/* Multi-process attribute sharding over NCCL (one process per GPU).  Rank 0 calls
 * gbdt_comm_unique_id and broadcasts the 128 bytes out of band (the Python binding uses
 * torch.distributed); every rank then calls gbdt_comm_init with the same id.  NCCL is loaded
 * at run time (dlopen "libnccl.so.2"); GBDT_E_NCCL if unavailable. */
gbdt_status gbdt_comm_unique_id(uint8_t id[128]);
gbdt_status gbdt_comm_init(int32_t rank, int32_t world, const uint8_t id[128], int32_t device,
                           gbdt_comm** out);
void gbdt_comm_free(gbdt_comm* c); /* NULL-safe; must outlive the datasets that use it */

/* Host-staged communicator with caller-supplied collectives, for testing the sharded path
 * without NCCL (e.g. two processes sharing one GPU, exchanging over torch.distributed/gloo).
 * The library synchronises its stream, copies the operand to a host buffer, calls the callback
 * with HOST pointers and copies the result back.  allgather: every rank contributes `bytes`
 * bytes, recv holds world * bytes in rank order.  allreduce_u8: element-wise uint8 sum in
 * place.  Callbacks return 0 on success (else GBDT_E_NCCL).  Same semantics as gbdt_comm_init
 * otherwise; `user` is passed through. */
typedef int (*gbdt_allgather_fn)(const void* send, void* recv, size_t bytes, void* user);
typedef int (*gbdt_allreduce_u8_fn)(void* buf, size_t n, void* user);
gbdt_status gbdt_comm_init_callbacks(int32_t rank, int32_t world, gbdt_allgather_fn allgather,
                                     gbdt_allreduce_u8_fn allreduce_u8, void* user, int32_t device,
                                     gbdt_comm** out);

/* Attribute ranges of a P-way sharding (host-only; no device is touched): shard i owns
 * attributes [bounds[i], bounds[i+1]), contiguous ranges balanced by stored entries
 * (col_counts[a] = entries of attribute a).  bounds: int32[P+1], caller-owned.  This is the
 * partition gbdt_load_csr uses for n_shards = P or a world of P ranks. */
gbdt_status gbdt_shard_ranges(int64_t n_cols, const int64_t* col_counts, int32_t P, int32_t* bounds);

void gbdt_dataset_free(gbdt_dataset* ds); /* NULL-safe */
void gbdt_model_free(gbdt_model* m);      /* NULL-safe */

/* Thread-local message of the last failing call on this thread ("" if none).  Valid until the
 * next call on this thread. */
const char* gbdt_last_error(void);

/* Number of kernel launches issued by the last gbdt_train on this thread (bench evidence). */
int64_t gbdt_last_launch_count(void);

#ifdef __cplusplus
}
#endif
#endif /* GBDT_H_ */
