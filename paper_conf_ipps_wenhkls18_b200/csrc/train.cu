// train.cu -- the per-tree / per-level hot path of GPU-GBDT on sm_100a.
//
//   a2 k_grad          SmartGD: yhat += eta*w[leaf], then g, h in fp64 (Eq. 1)
//   a3/a4/a5/a6 k_split_find   one pass over the level's attribute lists: segmented prefix sum of
//                      (g, h, count) per (node, attribute) segment (Fig. 1), gain of
//                      every distinct value at the end of its run (Eq. 2),
//                      missing values on both sides, per-piece argmax
//   a6 k_pick_* + k_decide  deterministic per-node argmax, split iff gain > max(gamma,0)
//                      (Alg. 1 l.14-21), tree emission, leaf weights (a9)
//   a7 k_mark + k_nodemap   instance -> child bitmap from the winning segment ("use the sorted
//                      values on that attribute to directly partition") and node map
//   a8 k_part_count / k_part_plan / k_part_scatter   order-preserving stable partition of every
//                      segment into its two children, entries of new leaves dropped
//
// Determinism: all fp64 sums use fixed association inside a tile; cross-tile carries are exact
// 128-bit fixed-point integer sums (levels.cu), so every attribute's prefix sums -- hence its
// gains -- are bit-identical whatever else is in the level buffer (other attributes, other
// shards, other runs).  The per-node argmax is over a strict
// total order (gain desc, attr asc, value desc, dir), so its result does not depend on the order
// in which pieces are reduced.
#include <nvtx3/nvToolsExt.h>

#include <algorithm>
#include <cstring>
#include <mutex>
#include <string>
#include <vector>

#include "kernels.cuh"

namespace gbdt {

namespace {

thread_local int64_t g_launches = 0;

// ============================================================================ a2: gradients
// SmartGD: the instances are in leaf nodes at the end of a tree, so the prediction is
// updated with the leaf weight of the node each instance ended in -- no tree traversal.
// Rows of the SmartGD-off ablation: the prediction before tree t is recomputed by traversing
// trees 0..t-1 over the instance's CSR row (the paper's baseline without SmartGD).
struct RowsArgs {
  const int64_t* indptr = nullptr;  // nullptr: SmartGD
  const int32_t* indices = nullptr;
  const float* values = nullptr;
  const gbdt_node* trees = nullptr;
  int64_t NH = 0;
  int t = 0;                         // trees already built
};
__device__ __forceinline__ double traverse_margin(const RowsArgs& R, int64_t i, double base, double eta) {
  double y = base;  // same operations in the same order as the SmartGD updates
  for (int u = 0; u < R.t; ++u)
    y = __dadd_rn(y, __dmul_rn(eta, tree_leaf_weight(R.trees + (int64_t)u * R.NH, R.indptr, R.indices, R.values, i)));
  return y;
}

// mode 0: built-in loss; 1: custom loss, prediction update only (the callback writes g, h);
// 2: custom loss, reduction of the callback's g, h only
// tidx: the tree index t on the device (nullptr: R.t); the previous tree's leaf weights are
// hweight + ((t + 1) & 1) * NH.
__global__ void k_grad(int64_t n, int loss, const int32_t* __restrict__ tidx, double eta, double base,
                       const float* __restrict__ y, const double* __restrict__ hweight, int64_t NH,
                       double* __restrict__ yhat, int32_t* __restrict__ pos,
                       double* __restrict__ gout, double* __restrict__ hout, int store_h,
                       double* __restrict__ partial, RowsArgs R, int mode, int* __restrict__ bad) {
  const int t = tidx ? *tidx : R.t;
  const int first = t == 0;
  const double* wprev = hweight + (size_t)((t + 1) & 1) * NH;
  R.t = t;
  double sg = 0.0, sh = 0.0, mg = 0.0, mh = 0.0, sl = 0.0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    double g, h;
    if (mode == 2) {
      g = gout[i];
      h = hout[i];
      if (!(isfinite(g) && isfinite(h) && h >= 0.0)) atomicOr(bad, 1);  // the callback's contract
    } else {
      double yh;
      if (R.indptr) yh = traverse_margin(R, i, base, eta);
      else yh = first ? base : __dadd_rn(yhat[i], __dmul_rn(eta, wprev[pos[i]]));
      yhat[i] = yh;
      pos[i] = 0;
      if (mode == 1) continue;
      const double yi = (double)y[i];
      // training loss at this margin (the model of the t trees before this one): (y - yhat)^2, or
      // the cross-entropy max(yhat, 0) - y yhat + log(1 + exp(-|yhat|)) (reported per tree)
      sl += loss == GBDT_LOSS_SQUARED ? (yi - yh) * (yi - yh)
                                      : fmax(yh, 0.0) - yi * yh + log1p(exp(-fabs(yh)));
    if (loss == GBDT_LOSS_SQUARED) {  // l = (y - yhat)^2: g = 2(yhat - y), h = 2 (R6)
      g = __dmul_rn(2.0, __dsub_rn(yh, yi));
      h = 2.0;
    } else {  // cross-entropy, Eq. 1: g = p - y, h = max(p(1-p), 1e-16) (reading R5)
      const double p = __ddiv_rn(1.0, __dadd_rn(1.0, exp(-yh)));
      g = __dsub_rn(p, yi);
      // h is stored (labels not all 0/1): p(1-p) itself; otherwise the split kernels recompute h
      // from the stored g (K1), so the node totals use that same form: q = g + y
      const double q = store_h ? p : __dadd_rn(g, yi);
      const double hh = __dmul_rn(q, __dsub_rn(1.0, q));
      h = hh > 1e-16 ? hh : 1e-16;
    }
    gout[i] = g;
    if (store_h) hout[i] = h;
    }
    sg += g;
    sh += h;
    mg = fmax(mg, fabs(g));
    mh = fmax(mh, fabs(h));
  }
  // fixed-shape block reduction (deterministic for a fixed grid)
  for (int o = 16; o; o >>= 1) {
    sg += __shfl_xor_sync(0xffffffffu, sg, o);
    sh += __shfl_xor_sync(0xffffffffu, sh, o);
    mg = fmax(mg, __shfl_xor_sync(0xffffffffu, mg, o));
    mh = fmax(mh, __shfl_xor_sync(0xffffffffu, mh, o));
    sl += __shfl_xor_sync(0xffffffffu, sl, o);
  }
  if (mode == 1) return;
  __shared__ double wg[32], wh[32], wmg[32], wmh[32], wl[32];
  if ((threadIdx.x & 31) == 0) {
    wg[threadIdx.x >> 5] = sg; wh[threadIdx.x >> 5] = sh;
    wmg[threadIdx.x >> 5] = mg; wmh[threadIdx.x >> 5] = mh; wl[threadIdx.x >> 5] = sl;
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double a = 0.0, b = 0.0, c = 0.0, e = 0.0, f = 0.0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) {
      a += wg[w]; b += wh[w]; c = fmax(c, wmg[w]); e = fmax(e, wmh[w]); f += wl[w];
    }
    partial[5 * blockIdx.x] = a;
    partial[5 * blockIdx.x + 1] = b;
    partial[5 * blockIdx.x + 2] = c;
    partial[5 * blockIdx.x + 3] = e;
    partial[5 * blockIdx.x + 4] = mode == 0 ? f : __longlong_as_double(0x7ff8000000000000ll);  // custom: unknown
  }
}

// fixed-point scale: value * 2^F < 2^125 for every |sum| <= n * max  (see levels.cu to_fx)
__device__ int fx_scale(double n, double mx) {
  const double M = n * mx;
  if (!(M > 0.0)) return 0;
  int e;
  frexp(M, &e);
  const int F = 125 - e;
  return F < -1000 ? -1000 : (F > 1000 ? 1000 : F);
}

// Root node totals + per-tree reset (single thread block).
__global__ void k_tree_begin(int nblk, const double* __restrict__ partial, int64_t n, double lam,
                             NodeTab root, int64_t NH, double* __restrict__ hweight,
                             uint8_t* __restrict__ hstate, gbdt_node* __restrict__ trees, int32_t* __restrict__ fx,
                             const int32_t* __restrict__ tidx, double* __restrict__ tloss) {
  const int t = *tidx;
  double* wcur = hweight + (size_t)(t & 1) * NH;
  gbdt_node* tree = trees + (size_t)t * NH;
  for (int64_t k = threadIdx.x; k < NH; k += blockDim.x) {
    wcur[k] = 0.0;
    hstate[k] = 0;
    gbdt_node z;
    z.heap_id = -1; z.is_leaf = 0; z.attr = -1; z.default_left = 0; z.split_value = 0.f;
    z.reserved = 0; z.gain = 0.0; z.G = 0.0; z.H = 0.0; z.weight = 0.0; z.count = 0;
    tree[k] = z;
  }
  // the k_grad block partials, reduced by the whole block in a fixed association (thread-strided
  // sums, a butterfly per warp, the warp totals in order): deterministic, and no longer one thread
  // walking ~1 k partials (84 us per tree on C2)
  __shared__ double red[5][32];
  {
    double G = 0.0, H = 0.0, mg = 0.0, mh = 0.0, L = 0.0;
    for (int b = threadIdx.x; b < nblk; b += blockDim.x) {
      G += partial[5 * b]; H += partial[5 * b + 1];
      mg = fmax(mg, partial[5 * b + 2]); mh = fmax(mh, partial[5 * b + 3]);
      L += partial[5 * b + 4];
    }
    for (int o = 16; o; o >>= 1) {
      G += __shfl_xor_sync(0xffffffffu, G, o);
      H += __shfl_xor_sync(0xffffffffu, H, o);
      mg = fmax(mg, __shfl_xor_sync(0xffffffffu, mg, o));
      mh = fmax(mh, __shfl_xor_sync(0xffffffffu, mh, o));
      L += __shfl_xor_sync(0xffffffffu, L, o);
    }
    if ((threadIdx.x & 31) == 0) {
      const int w = threadIdx.x >> 5;
      red[0][w] = G; red[1][w] = H; red[2][w] = mg; red[3][w] = mh; red[4][w] = L;
    }
  }
  __syncthreads();
  if (threadIdx.x == 0) {
    double G = 0.0, H = 0.0, mg = 0.0, mh = 0.0, L = 0.0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) {
      G += red[0][w]; H += red[1][w]; mg = fmax(mg, red[2][w]); mh = fmax(mh, red[3][w]); L += red[4][w];
    }
    tloss[t] = L / (double)n;  // mean training loss of the model of trees 0 .. t-1
    fx[0] = fx_scale((double)n, mg);
    fx[1] = fx_scale((double)n, mh);
    *root.K = 1;
    root.heap[0] = 0;
    root.G[0] = G;
    root.H[0] = H;
    root.cnt[0] = (int32_t)n;
    root.pterm[0] = parent_term(G, H, lam);
  }
}

__global__ void k_tree_end(int32_t* __restrict__ tidx) { *tidx += 1; }

__global__ void k_level_begin(int* __restrict__ epoch, int* __restrict__ counters, int ncounters,
                              int* __restrict__ nrec, int nshard, const int32_t* __restrict__ Kp,
                              unsigned long long* __restrict__ gkey, unsigned long long* __restrict__ tkey,
                              int Kcap) {
  if (threadIdx.x == 0) *epoch = *epoch + 1;
  for (int i = threadIdx.x; i < ncounters; i += blockDim.x) counters[i] = 0;
  for (int i = threadIdx.x; i < nshard; i += blockDim.x) nrec[i] = 0;
  const int K = *Kp;
  for (int i = threadIdx.x; i < nshard * Kcap; i += blockDim.x) {
    if (i % Kcap < K) { gkey[i] = 0ull; tkey[i] = ~0ull; }
  }
}

// ============================================================================ a6: decide
__global__ void k_pick_tie(const Rec* __restrict__ rec, const int* __restrict__ nrec,
                           const unsigned long long* __restrict__ gkey,
                           unsigned long long* __restrict__ tkey) {
  const int n = *nrec;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const Rec& r = rec[i];
    if (gain_key(r.gain) == gkey[r.node]) atomicMin(tkey + r.node, tie_key(r.attr, r.value, r.dir));
  }
}

__global__ void k_pick_best(const Rec* __restrict__ rec, const int* __restrict__ nrec,
                            const unsigned long long* __restrict__ gkey,
                            const unsigned long long* __restrict__ tkey, Rec* __restrict__ best) {
  const int n = *nrec;
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x) {
    const Rec r = rec[i];
    if (gain_key(r.gain) == gkey[r.node] && tie_key(r.attr, r.value, r.dir) == tkey[r.node]) best[r.node] = r;
  }
}

__device__ unsigned long long block_exscan_u64(unsigned long long x, unsigned long long& total) {
  __shared__ unsigned long long ws[32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  unsigned long long incl = x;
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long y = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) ws[w] = incl;
  __syncthreads();
  if (w == 0) {
    unsigned long long s = lane < nw ? ws[lane] : 0ull, si = s;
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(0xffffffffu, si, o);
      if (lane >= o) si += y;
    }
    if (lane < nw) ws[lane] = si - s;
  }
  __syncthreads();
  const unsigned long long ex = ws[w] + incl - x;
  // total = exclusive of the last thread + its value; fetch via the last warp's slot
  __shared__ unsigned long long tot;
  if (threadIdx.x == blockDim.x - 1) tot = ex + x;
  __syncthreads();
  total = tot;
  __syncthreads();
  return ex;
}

struct DecideArgs {
  NodeTab cur, nxt;
  const Rec* best_all;  // [nshard][Kcap]
  int nshard, Kcap;
  const int* epochp;
  double lam, thr;
  int last_level;
  int32_t* cidx;        // [Kcap] next-level index of the high child, -1 if not split
  Rec* winner;          // [Kcap]
  uint8_t* hstate;      // by heap id: 1 split at this level, 2 leaf
  uint8_t* hdef;        // default side: 1 high
  double* hweight;      // by heap id, two trees (this one: + (t & 1) * NH)
  gbdt_node* trees;     // all trees (this one: + t * NH)
  gbdt_node* tree;      // set by k_decide
  const int32_t* tidx;  // t
  int64_t NH;
};

__device__ void write_leaf(const DecideArgs& A, int h, double G, double H, long long cnt) {
  const double w = __ddiv_rn(-G, __dadd_rn(H, A.lam));  // reading R3: w = -G/(H+lambda)
  gbdt_node nd;
  nd.heap_id = h; nd.is_leaf = 1; nd.attr = -1; nd.default_left = 0; nd.split_value = 0.f;
  nd.reserved = 0; nd.gain = 0.0; nd.G = G; nd.H = H; nd.weight = w; nd.count = cnt;
  A.tree[h] = nd;
  A.hweight[h] = w;
  A.hstate[h] = 2;
}

// Single thread block: merge the shards' node bests (strict total order), decide, emit.
__global__ void k_decide(DecideArgs A) {
  {
    const int t = *A.tidx;
    A.hweight += (size_t)(t & 1) * A.NH;
    A.tree = A.trees + (size_t)t * A.NH;
  }
  const int K = *A.cur.K;
  const int epoch = *A.epochp;
  unsigned long long carry = 0;
  for (int base = 0; base < K; base += blockDim.x) {
    const int j = base + threadIdx.x;
    int split = 0;
    Rec b;
    if (j < K) {
      bool found = false;
      unsigned long long bg = 0, bt = 0;
      for (int s = 0; s < A.nshard; ++s) {
        const Rec r = A.best_all[(size_t)s * A.Kcap + j];
        if (r.epoch != epoch) continue;
        const unsigned long long rg = gain_key(r.gain), rt = tie_key(r.attr, r.value, r.dir);
        if (!found || rg > bg || (rg == bg && rt < bt)) { b = r; bg = rg; bt = rt; found = true; }
      }
      split = found && b.gain > A.thr;  // Alg. 1 l.15-17 (strict), reading R2
    }
    unsigned long long tot;
    const unsigned long long rank = block_exscan_u64((unsigned long long)split, tot);
    if (j < K) {
      const int h = A.cur.heap[j];
      const double G = A.cur.G[j], H = A.cur.H[j];
      const int cnt = A.cur.cnt[j];
      if (!split) {
        A.cidx[j] = -1;
        write_leaf(A, h, G, H, cnt);
      } else {
        const int c = 2 * (int)(carry + rank);
        A.cidx[j] = c;
        A.winner[j] = b;
        A.hstate[h] = 1;
        A.hdef[h] = (uint8_t)b.dir;
        gbdt_node nd;
        nd.heap_id = h; nd.is_leaf = 0; nd.attr = b.attr; nd.default_left = b.dir;
        nd.split_value = b.value; nd.reserved = 0; nd.gain = b.gain; nd.G = G; nd.H = H;
        nd.weight = 0.0; nd.count = cnt;
        A.tree[h] = nd;
        const double GH = b.GL, HH = b.HL;
        const double GLo = G - b.GL, HLo = H - b.HL;
        const int cH = (int)b.cntL, cLo = cnt - (int)b.cntL;
        if (A.last_level) {
          write_leaf(A, 2 * h + 1, GH, HH, cH);
          write_leaf(A, 2 * h + 2, GLo, HLo, cLo);
        } else {
          A.nxt.heap[c] = 2 * h + 1; A.nxt.G[c] = GH; A.nxt.H[c] = HH; A.nxt.cnt[c] = cH;
          A.nxt.pterm[c] = parent_term(GH, HH, A.lam);
          A.nxt.heap[c + 1] = 2 * h + 2; A.nxt.G[c + 1] = GLo; A.nxt.H[c + 1] = HLo; A.nxt.cnt[c + 1] = cLo;
          A.nxt.pterm[c + 1] = parent_term(GLo, HLo, A.lam);
          gbdt_node ch;
          ch.heap_id = 2 * h + 1; ch.is_leaf = 0; ch.attr = -1; ch.default_left = 0; ch.split_value = 0.f;
          ch.reserved = 0; ch.gain = 0.0; ch.G = GH; ch.H = HH; ch.weight = 0.0; ch.count = cH;
          A.tree[2 * h + 1] = ch;
          ch.heap_id = 2 * h + 2; ch.G = GLo; ch.H = HLo; ch.count = cLo;
          A.tree[2 * h + 2] = ch;
        }
      }
    }
    carry += tot;
  }
  if (threadIdx.x == 0) *A.nxt.K = A.last_level ? 0 : (int)(2 * carry);
}

// ============================================================================ a7: node map
__global__ void k_mark(const int32_t* __restrict__ Kp, const int32_t* __restrict__ cidx,
                       const Rec* __restrict__ winner, int shard, int a_base, Tables tb,
                       const int32_t* __restrict__ ins, uint32_t* __restrict__ bits,
                       const uint8_t* __restrict__ sflag, ShortList S) {
  const int K = *Kp;
  const int j = blockIdx.y;
  if (j >= K || cidx[j] < 0) return;
  const Rec& w = winner[j];
  if (w.shard != shard) return;
  if (S.inplace && S.jl && sflag && sflag[w.attr - a_base]) {
    // an in-place short list (not partitioned): node j's entries are those carrying j, in value
    // order; the high side is every one up to the winner's position (root positions)
    if (blockIdx.x != 0) return;
    const int a = w.attr - a_base;
    const long long p0 = S.cs0[a], L = S.cl0[a];
    for (long long q = threadIdx.x; q < L; q += blockDim.x) {
      const long long p = p0 + q;
      if ((int)S.jl[p] != j) continue;
      if ((int)(p <= w.pos) != w.dir) {
        const int i = S.ins0[p];
        atomicOr(bits + (i >> 5), 1u << (i & 31));
      }
    }
    return;
  }
  const long long s = (long long)(w.attr - a_base) * K + j;
  const long long s0 = tb.seg_start[s], n = tb.seg_cnt[s];
  const int defhi = w.dir;
  for (long long q = (long long)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (long long)gridDim.x * blockDim.x) {
    const long long p = s0 + q;
    const int high = p <= w.pos;   // prefix of the descending list = values >= split value
    if (high != defhi) {  // goes to the non-default side: bit i of the n-bit map (multi-GPU: OR-allreduced)
      const int i = ins[p];
      atomicOr(bits + (i >> 5), 1u << (i & 31));
    }
  }
}

// side[i]: 0 (node became a leaf), 1 (high child), 2 (low child); hbit: bit i = [side[i] == 1],
// packed by warp ballots (the dense partition count gathers these 1.4 MB instead of 11 MB)
__global__ void k_nodemap(int64_t n, const uint32_t* __restrict__ bits, const uint8_t* __restrict__ hstate,
                          const uint8_t* __restrict__ hdef, int32_t* __restrict__ pos,
                          uint8_t* __restrict__ side, uint32_t* __restrict__ hbit) {
  const int64_t n32 = (n + 31) & ~int64_t(31);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n32; i += (int64_t)gridDim.x * blockDim.x) {
    uint8_t sd = 0;
    if (i < n) {
      const int h = pos[i];
      if (hstate[h] == 1) {
        const int defhi = hdef[h];
        const int hi = ((bits[i >> 5] >> (i & 31)) & 1u) ? !defhi : defhi;
        pos[i] = hi ? 2 * h + 1 : 2 * h + 2;
        sd = hi ? 1 : 2;
      }
      side[i] = sd;
    }
    const unsigned b = __ballot_sync(0xffffffffu, sd == 1);
    if ((threadIdx.x & 31) == 0) hbit[i >> 5] = b;
  }
}

// Mean training loss of the final model (after the last tree's SmartGD update), same terms and
// block-then-ordered association as k_grad's
__global__ void k_loss_partial(int64_t n, int loss, const double* __restrict__ yhat, const float* __restrict__ y,
                               double* __restrict__ partial) {
  double sl = 0.0;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const double yh = yhat[i], yi = (double)y[i];
    sl += loss == GBDT_LOSS_SQUARED ? (yi - yh) * (yi - yh) : fmax(yh, 0.0) - yi * yh + log1p(exp(-fabs(yh)));
  }
  for (int o = 16; o; o >>= 1) sl += __shfl_xor_sync(0xffffffffu, sl, o);
  __shared__ double wl[32];
  if ((threadIdx.x & 31) == 0) wl[threadIdx.x >> 5] = sl;
  __syncthreads();
  if (threadIdx.x == 0) {
    double f = 0.0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) f += wl[w];
    partial[5 * blockIdx.x + 4] = f;
  }
}
__global__ void k_loss_final(int nblk, const double* __restrict__ partial, int64_t n, int custom,
                             double* __restrict__ out) {
  double L = 0.0;
  for (int b = 0; b < nblk; ++b) L += partial[5 * b + 4];
  *out = custom ? __longlong_as_double(0x7ff8000000000000ll) : L / (double)n;
}

__global__ void k_apply(int64_t n, double eta, const double* __restrict__ w, const int32_t* __restrict__ pos,
                        double* __restrict__ yhat) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    yhat[i] = __dadd_rn(yhat[i], __dmul_rn(eta, w[pos[i]]));
}

}  // namespace

void count_launch(int k) { g_launches += k; }
int64_t launches_get() { return g_launches; }
void launches_reset() { g_launches = 0; }

// ============================================================================ host side
namespace {

struct Carve {
  char* base;
  size_t off = 0;
  template <class T> T* take(size_t n) {
    off = (off + 255) & ~size_t(255);
    T* p = reinterpret_cast<T*>(base + off);
    off += n * sizeof(T);
    return p;
  }
};

constexpr int kShortLevels = 6;  // levels with K <= 32 (2^5): the short path's node tables

struct ShardWork {
  DBuf mem;
  Tables tab[2];
  DBuf lists;                 // g-lists (+ h-lists) of two levels, entry-aligned with val/ins
  double *glist[2], *hlist[2];
  uint8_t* slist;
  unsigned long long *cagg, *carry;   // [C0][5]
  unsigned long long *ccnt, *cpre;    // [C0][2]
  unsigned long long* sgrp;           // scan scratch
  unsigned groups;
  Rec* rec;
  ChunkDesc* desc;
  int32_t* genlist;
  int32_t* segEnd;
  int* nrec;
  unsigned long long *gkey, *tkey;
  int32_t *segH, *segL;
  unsigned long long* seg_pre;
  int64_t *out_hi, *out_lo, *len_tmp;
  double *segPG, *segPH;
  int* counters;  // [4]
  // RLE (a8): run tables of two levels live in tab[b]; scratch of the direct run split
  DBuf runs;
  int32_t* run_seg = nullptr;
  unsigned long long *run_hl = nullptr, *rcnt = nullptr, *rfl = nullptr, *rsgrp = nullptr;
  int32_t* Rp1 = nullptr;
  unsigned rgroups = 1;
  unsigned long long* racc = nullptr;  // RLE split on runs: [Rcap][5] exact (g, h) per run (scan records)
  unsigned long long* rcar = nullptr;  //   their exclusive segmented prefixes (fp64 carries)
  unsigned long long* rsg5 = nullptr;  //   scan scratch
  uint32_t* enc_cnt = nullptr;   // RLE split ablation: runs per next-level chunk
  uint32_t* enc_bits = nullptr;  //   and the next level's segment-start bitmap
  // fused dense levels: plans of two levels, per-tile records / carries / side bits
  DBuf fz;
  FusedPlan* fplan[2] = {nullptr, nullptr};
  void* tilemem = nullptr;
  int64_t tiles = 0;
  // attribute-parallel partition plan
  unsigned long long *pel = nullptr, *pgrp = nullptr;
  int32_t* mp1 = nullptr;
  unsigned pgroups = 1;
  // short-attribute path (levels.cu k_short_*): the attributes, their flags, the chunk kernels'
  // chunk lists of the root and of the two level tables
  DBuf shortmem;
  ShortList sl;
  int32_t* longa = nullptr;  // the attributes not on the short path
  int nlong = 0;
  uint8_t* sflag = nullptr;
  uint8_t* jl[2] = {nullptr, nullptr};  // node index of each short-list entry, two levels
  DBuf shortg;                           // in-place mode: the short lists' g (h) lists
  // the level's short-path arguments (levels 0..kShortLevels-1, where K <= 32), else none
  ShortList level_sl(int lvl) const {
    ShortList r = sl;
    if (lvl >= kShortLevels) { r.n = 0; r.nb = 0; r.inplace = 0; return r; }
    if (sl.inplace) {  // one node-index list, updated in place
      r.jl = lvl == 0 ? nullptr : jl[0];
      r.jl_out = jl[0];
      return r;
    }
    r.jl = lvl == 0 ? nullptr : jl[lvl & 1];
    r.jl_out = lvl + 1 < kShortLevels ? jl[(lvl + 1) & 1] : nullptr;
    return r;
  }
  const uint8_t* level_flag(int lvl) const { return (sl.nb && lvl < kShortLevels) ? sflag : nullptr; }
  Tables root;  // the shard's root tables (+ the root chunk list on the short path)
};

// NVTX names of the phases (host-side ranges for nsys / ncu --nvtx; no-ops without a tool)
const char* const kPhaseName[GBDT_N_PHASES] = {"grad", "split_find", "decide", "nodemap", "partition", "comm",
                                               "total", "k_chunk_agg", "k_split", "k_count", "k_scatter",
                                               "k_fused"};

struct PhaseTimer {
  bool on = false;
  bool nvtx = false;  // phase ranges (the outer timer only, so the ranges nest)
  cudaStream_t st = nullptr;
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> ev;
  int cur = -1;
  cudaEvent_t e0 = nullptr;
  void begin(int phase) {
    if (nvtx) nvtxRangePushA(kPhaseName[phase]);
    if (!on) return;
    cudaEvent_t a;
    GBDT_CUDA(cudaEventCreate(&a));
    GBDT_CUDA(cudaEventRecord(a, st));
    cur = phase;
    e0 = a;
  }
  void end() {
    if (nvtx) nvtxRangePop();
    if (!on) return;
    cudaEvent_t b;
    GBDT_CUDA(cudaEventCreate(&b));
    GBDT_CUDA(cudaEventRecord(b, st));
    ev.push_back({cur, {e0, b}});
  }
  void collect(double* ms) {
    for (auto& x : ev) {
      float t = 0;
      GBDT_CUDA(cudaEventElapsedTime(&t, x.second.first, x.second.second));
      ms[x.first] += t;
      cudaEventDestroy(x.second.first);
      cudaEventDestroy(x.second.second);
    }
    ev.clear();
  }
};

}  // namespace

// sum of the level's attribute list lengths (profile = 1 only)
__global__ void k_level_entries(const int64_t* col_len, int m, unsigned long long* out) {
  unsigned long long s = 0;
  for (int a = blockIdx.x * blockDim.x + threadIdx.x; a < m; a += gridDim.x * blockDim.x) s += (unsigned long long)col_len[a];
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(out, s);
}

// Level kernels are configured once per device (smem attributes, persistent grid sizes); safe
// when several host threads train different handles at once.
static LevelKernels& level_kernels(int device) {
  static LevelKernels lk[kMaxDevices];
  static std::once_flag once[kMaxDevices];
  static std::string err[kMaxDevices];
  static gbdt_status est[kMaxDevices];
  if (device < 0 || device >= kMaxDevices) fail(GBDT_E_RANGE, "device ordinal >= " + std::to_string(kMaxDevices));
  std::call_once(once[device], [device] {
    try {
      lk[device].init(device);
      est[device] = GBDT_OK;
    } catch (const Error& e) {
      est[device] = e.st;
      err[device] = e.msg;
    }
  });
  if (est[device] != GBDT_OK) fail(est[device], err[device]);
  return lk[device];
}

void train(Dataset& ds, const gbdt_params& P, Model& model, double* margin_out) {
  GBDT_CUDA(cudaSetDevice(ds.device));
  cudaStream_t st = ds.stream;
  launches_reset();
  LevelKernels& LK = level_kernels(ds.device);
  const int d = P.max_depth;
  const int64_t NH = (int64_t(1) << (d + 1)) - 1;
  const int Kcap = 1 << (d - 1);
  const int64_t n = ds.n;
  const int nloc = (int)ds.shards.size();
  const int nsh = ds.n_total_shards;
  const int sms = LK.sms;
  // gradient storage mode (kernels.cuh): squared -> h == 2; logistic with 0/1 labels -> h(g)
  const int hmode = P.loss == GBDT_LOSS_SQUARED ? kHConst2
                    : (P.loss == GBDT_LOSS_LOGISTIC && ds.binary_labels ? kHFromG : kHGather);
  const bool custom = P.loss == GBDT_LOSS_CUSTOM;
  RowsArgs rows;  // SmartGD-off ablation
  if (P.smartgd_off) {
    rows.indptr = ds.rows_ptr.as<int64_t>(); rows.indices = ds.rows_idx.as<int32_t>();
    rows.values = ds.rows_val.as<float>(); rows.NH = NH;
  }
  const unsigned inst_grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), (int64_t)sms * 8));
  const int grad_blocks = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), (int64_t)sms * 4));
  const int64_t npad = (n + 8) & ~int64_t(3);

  // ---------------------------------------------------------------- per-device state
  auto sz_dev = [&](Carve& c) {
    c.take<double>(n); c.take<double>(hmode == kHGather ? n : 1); c.take<double>(n); c.take<int32_t>(n);
    c.take<uint8_t>(npad); c.take<uint32_t>((size_t)(n + 31) / 32 + 1);
    c.take<double>(2 * NH); c.take<uint8_t>(NH); c.take<uint8_t>(NH);
    c.take<gbdt_node>((size_t)P.n_trees * NH); c.take<double>(5 * grad_blocks); c.take<int32_t>(2);
    c.take<double>((size_t)P.n_trees + 1);
    for (int b = 0; b < 2; ++b) { c.take<int32_t>(1); c.take<int32_t>(Kcap); c.take<double>(Kcap); c.take<double>(Kcap); c.take<int32_t>(Kcap); c.take<double>(Kcap); }
    c.take<int32_t>(Kcap); c.take<Rec>(Kcap); c.take<Rec>((size_t)nsh * Kcap); c.take<int>(1);
    c.take<unsigned long long>((size_t)nloc * Kcap); c.take<unsigned long long>((size_t)nloc * Kcap);
    c.take<int>(nloc);
    c.take<unsigned long long>(16);
    c.take<int32_t>(4);
    c.take<uint32_t>((size_t)(n + 31) / 32 + 1);
    c.take<uint32_t>((size_t)(n + 31) / 32 + 1);
  };
  Carve probe{nullptr};
  sz_dev(probe);
  DBuf dmem(probe.off + 1024, st);
  GBDT_CUDA(cudaMemsetAsync(dmem.p, 0, dmem.bytes, st));
  Carve c{dmem.as<char>()};
  double* gv = c.take<double>(n);
  double* hv = c.take<double>(hmode == kHGather ? n : 1);
  double* yhat = c.take<double>(n);
  int32_t* pos = c.take<int32_t>(n);
  uint8_t* side = c.take<uint8_t>(npad);
  uint32_t* bits = c.take<uint32_t>((size_t)(n + 31) / 32 + 1);  // instance -> non-default side (n bits)
  double* hweight = c.take<double>(2 * NH);
  uint8_t* hstate = c.take<uint8_t>(NH);
  uint8_t* hdef = c.take<uint8_t>(NH);
  gbdt_node* trees = c.take<gbdt_node>((size_t)P.n_trees * NH);
  double* partial = c.take<double>(5 * grad_blocks);
  int32_t* fxs = c.take<int32_t>(2);
  double* tloss = c.take<double>((size_t)P.n_trees + 1);  // mean training loss after 0 .. T trees
  NodeTab nt[2];
  for (int b = 0; b < 2; ++b) {
    nt[b].K = c.take<int32_t>(1); nt[b].heap = c.take<int32_t>(Kcap); nt[b].G = c.take<double>(Kcap);
    nt[b].H = c.take<double>(Kcap); nt[b].cnt = c.take<int32_t>(Kcap); nt[b].pterm = c.take<double>(Kcap);
  }
  int32_t* cidx = c.take<int32_t>(Kcap);
  Rec* winner = c.take<Rec>(Kcap);
  Rec* best_all = c.take<Rec>((size_t)nsh * Kcap);
  int* epoch = c.take<int>(1);
  unsigned long long* gkey = c.take<unsigned long long>((size_t)nloc * Kcap);
  unsigned long long* tkey = c.take<unsigned long long>((size_t)nloc * Kcap);
  int* nrec = c.take<int>(nloc);
  unsigned long long* lent = c.take<unsigned long long>(16);  // entries scanned per level (profile)
  int32_t* tidx = c.take<int32_t>(4);  // index of the tree being built (device side, for graph replays)
  uint32_t* hbit = c.take<uint32_t>((size_t)(n + 31) / 32 + 1);  // instance -> high child bit
  uint32_t* hbit2 = c.take<uint32_t>((size_t)(n + 31) / 32 + 1);  // the fused path's second level
  uint32_t* hbitF[2] = {hbit, hbit2};

  // Fused dense levels (fused.cu): no missing values, g-list only, K <= kFusedMaxK at the last
  // partitioned level, plain lists with the dense root layout (attribute a at a * pad4(n))
  bool fused = !ds.has_missing && hmode != kHGather && d >= 2 && d <= 8;
  for (auto& shp : ds.shards) {
    const Shard& sh = *shp;
    if (sh.rle) fused = false;
    for (int a = 0; a < sh.m && fused; ++a)
      if (sh.h_col_len[a] != n || sh.h_col_start[a] != (int64_t)a * pad4(n)) fused = false;
  }
  // Test hook (kernel-level invariants): GBDT_CAPTURE_LEVEL=l copies level l's lists,
  // segment tables and runs of tree 0 to the model (gbdt_model_export_level); eager launches only
  int cap_level = -1;
  if (const char* cl = getenv("GBDT_CAPTURE_LEVEL")) cap_level = atoi(cl);
  if (cap_level >= 0) fused = false;
  {  // opt-in while the fused pass is being tuned (GBDT_FUSED=1)
    const char* fe = getenv("GBDT_FUSED");
    fused = fused && fe && fe[0] != '0';
  }
  // RLE shards without missing values find splits over the runs (levels.cu k_run_split);
  // GBDT_RUNSPLIT=0 keeps the per-entry scan of the plain lists (A/B and cross-check)
  bool runsplit = !ds.has_missing;
  if (const char* rse = getenv("GBDT_RUNSPLIT")) runsplit = runsplit && rse[0] != '0';

  // ---------------------------------------------------------------- per-shard state
  std::vector<ShardWork> sw(nloc);
  for (int li = 0; li < nloc; ++li) {
    Shard& sh = *ds.shards[li];
    ShardWork& w = sw[li];
    const int m = sh.m;
    const int64_t S = (int64_t)m * Kcap;
    const int64_t C0 = std::max(sh.C0, 1);
    // node-best records per level: one per CTA and node (K <= 32), else one per chunk and segment
    const int64_t R = (int64_t)(LK.grid_fast[2][1] + LK.grid_fast[1][1] + LK.grid_fast[0][1] + LK.grid_gen + LK.grid_short +
                                LK.grid_sl) * 64 +
                      (int64_t)LK.grid_fused * 2 * kFusedMaxK + 2 * C0 + S + 64;
    auto sz = [&](Carve& q) {
      for (int b = 0; b < 2; ++b) {
        q.take<int64_t>(m + 1); q.take<int64_t>(m); q.take<int32_t>(m + 1); q.take<int32_t>(m + 1);
        q.take<int64_t>(S); q.take<int64_t>(S); q.take<int32_t>(1); q.take<int32_t>(1); q.take<int32_t>(C0);
      }
      q.take<unsigned long long>(5 * C0); q.take<unsigned long long>(5 * C0);
      q.take<unsigned long long>(2 * C0); q.take<unsigned long long>(2 * C0);
      q.take<unsigned long long>(5 * (size_t)LevelKernels::scan_groups(C0) + 8);
      q.take<Rec>(R); q.take<ChunkDesc>(C0); q.take<int32_t>(C0); q.take<int32_t>(S);
      q.take<int32_t>(S); q.take<int32_t>(S); q.take<unsigned long long>(S); q.take<int64_t>(S); q.take<int64_t>(S);
      q.take<int64_t>(m); q.take<double>(S); q.take<double>(S); q.take<int>(4);
      q.take<unsigned long long>(2 * (size_t)(m + 1)); q.take<unsigned long long>(2 * (size_t)LevelKernels::scan_groups(m + 1) + 8);
      q.take<int32_t>(1);
    };
    Carve pq{nullptr};
    sz(pq);
    w.mem.alloc(pq.off + 1024, st);
    GBDT_CUDA(cudaMemsetAsync(w.mem.p, 0, w.mem.bytes, st));
    Carve q{w.mem.as<char>()};
    for (int b = 0; b < 2; ++b) {
      w.tab[b].col_start = q.take<int64_t>(m + 1); w.tab[b].col_len = q.take<int64_t>(m);
      w.tab[b].tile_start = q.take<int32_t>(m + 1); w.tab[b].chunk_start = q.take<int32_t>(m + 1);
      w.tab[b].seg_start = q.take<int64_t>(S); w.tab[b].seg_cnt = q.take<int64_t>(S);
      w.tab[b].T = q.take<int32_t>(1); w.tab[b].C = q.take<int32_t>(1);
      w.tab[b].chunk_attr = q.take<int32_t>(C0);
    }
    w.cagg = q.take<unsigned long long>(5 * C0); w.carry = q.take<unsigned long long>(5 * C0);
    w.ccnt = q.take<unsigned long long>(2 * C0); w.cpre = q.take<unsigned long long>(2 * C0);
    w.groups = LevelKernels::scan_groups(C0);
    w.sgrp = q.take<unsigned long long>(5 * (size_t)w.groups + 8);
    const int nl = hmode == kHGather ? 4 : 2;
    w.lists.alloc((size_t)sh.cap * 8 * nl + (size_t)sh.cap + 64, st);
    w.slist = reinterpret_cast<uint8_t*>(w.lists.as<double>() + (size_t)sh.cap * nl);
    for (int b = 0; b < 2; ++b) {
      w.glist[b] = w.lists.as<double>() + (size_t)b * sh.cap;
      w.hlist[b] = hmode == kHGather ? w.lists.as<double>() + (size_t)(2 + b) * sh.cap : nullptr;
    }
    w.rec = q.take<Rec>(R);
    w.desc = q.take<ChunkDesc>(C0);
    w.genlist = q.take<int32_t>(C0);
    w.segEnd = q.take<int32_t>(S);
    w.segH = q.take<int32_t>(S); w.segL = q.take<int32_t>(S);
    w.seg_pre = q.take<unsigned long long>(S);
    w.out_hi = q.take<int64_t>(S); w.out_lo = q.take<int64_t>(S);
    w.len_tmp = q.take<int64_t>(m);
    w.segPG = q.take<double>(S); w.segPH = q.take<double>(S);
    w.counters = q.take<int>(4);
    w.pgroups = LevelKernels::scan_groups(m + 1);
    w.pel = q.take<unsigned long long>(2 * (size_t)(m + 1));
    w.pgrp = q.take<unsigned long long>(2 * (size_t)w.pgroups + 8);
    w.mp1 = q.take<int32_t>(1);
    {
      const int32_t mp1 = m + 1;
      GBDT_CUDA(cudaMemcpyAsync(w.mp1, &mp1, 4, cudaMemcpyHostToDevice, st));
      GBDT_CUDA(cudaStreamSynchronize(st));
    }
    if (sh.rle) {
      // child runs: every run splits in at most two, and there are never more runs than entries
      const int64_t Rcap = std::max<int64_t>(1, std::min<int64_t>(sh.runs * Kcap, sh.cap));
      w.rgroups = LevelKernels::scan_groups(Rcap + 1);
      auto rz = [&](Carve& q) {
        for (int b = 0; b < 2; ++b) {
          q.take<float>(Rcap); q.take<int32_t>(Rcap); q.take<int64_t>(Rcap); q.take<int32_t>(S + 1); q.take<int32_t>(1);
          q.take<int32_t>(C0 + 1);
        }
        q.take<int32_t>(Rcap); q.take<unsigned long long>(Rcap); q.take<unsigned long long>(2 * Rcap);
        q.take<unsigned long long>(2 * (Rcap + 1)); q.take<int32_t>(1);
        q.take<unsigned long long>(2 * (size_t)w.rgroups + 8);
        q.take<uint32_t>((size_t)C0 + 2);
        q.take<uint32_t>((size_t)sh.cap / 32 + 2);
        q.take<unsigned long long>(5 * (size_t)Rcap); q.take<unsigned long long>(5 * (size_t)Rcap);
        q.take<unsigned long long>(5 * (size_t)w.rgroups + 8);
      };
      Carve rp{nullptr};
      rz(rp);
      w.runs.alloc(rp.off + 1024, st);
      GBDT_CUDA(cudaMemsetAsync(w.runs.p, 0, w.runs.bytes, st));
      Carve r{w.runs.as<char>()};
      for (int b = 0; b < 2; ++b) {
        w.tab[b].run_val = r.take<float>(Rcap); w.tab[b].run_len = r.take<int32_t>(Rcap);
        w.tab[b].run_pos = r.take<int64_t>(Rcap); w.tab[b].seg_run = r.take<int32_t>(S + 1);
        w.tab[b].R = r.take<int32_t>(1);
        w.tab[b].run_chunk = r.take<int32_t>(C0 + 1);
      }
      w.run_seg = r.take<int32_t>(Rcap); w.run_hl = r.take<unsigned long long>(Rcap);
      w.rcnt = r.take<unsigned long long>(2 * Rcap); w.rfl = r.take<unsigned long long>(2 * (Rcap + 1));
      w.Rp1 = r.take<int32_t>(1); w.rsgrp = r.take<unsigned long long>(2 * (size_t)w.rgroups + 8);
      w.enc_cnt = r.take<uint32_t>((size_t)C0 + 2);
      w.enc_bits = r.take<uint32_t>((size_t)sh.cap / 32 + 2);
      w.racc = r.take<unsigned long long>(5 * (size_t)Rcap); w.rcar = r.take<unsigned long long>(5 * (size_t)Rcap);
      w.rsg5 = r.take<unsigned long long>(5 * (size_t)w.rgroups + 8);
    }
    if (fused && m > 0) {
      w.tiles = fused_tiles(n, m);
      const size_t tb = fused_tile_bytes(w.tiles);
      w.fz.alloc(2 * sizeof(FusedPlan) + 1024 + tb, st);
      GBDT_CUDA(cudaMemsetAsync(w.fz.p, 0, w.fz.bytes, st));
      Carve f{w.fz.as<char>()};
      w.fplan[0] = f.take<FusedPlan>(1);
      w.fplan[1] = f.take<FusedPlan>(1);
      w.tilemem = f.take<char>(tb);
    }
    // Short path (levels.cu k_short_*): sparse lists (missing values) kept as plain lists, the
    // attributes whose root list has at most 32 entries (GBDT_SHORT=0 turns the path off)
    w.root = sh.root;
    {
      const char* se = getenv("GBDT_SHORT");
      const int64_t short_max = 32;
      const bool on = (se ? se[0] != '0' : true) && ds.has_missing && !sh.rle && !ds.dense && m > 0;
      std::vector<int32_t> attrs;
      if (on) {
        // longest first (a counting sort by root length), so the warps' loads even out
        std::vector<int64_t> bucket((size_t)short_max + 2, 0);
        for (int a = 0; a < m; ++a) {
          const int64_t L = sh.h_col_len[a];
          if (L > 0 && L <= short_max) ++bucket[(size_t)(short_max - L)];
        }
        int64_t acc = 0;
        for (auto& b : bucket) { const int64_t x = b; b = acc; acc += x; }
        attrs.resize((size_t)acc);
        for (int a = 0; a < m; ++a) {
          const int64_t L = sh.h_col_len[a];
          if (L > 0 && L <= short_max) attrs[(size_t)bucket[(size_t)(short_max - L)]++] = a;
        }
      }
      if (!attrs.empty()) {
        std::vector<uint8_t> flag((size_t)m, 0);
        for (int32_t a : attrs) flag[(size_t)a] = 1;
        std::vector<int32_t> longa;  // the other attributes (k_seg_totals)
        for (int a = 0; a < m; ++a)
          if (!flag[(size_t)a]) longa.push_back(a);
        std::vector<int32_t> lc;  // root chunks of the other attributes (chunk_start as build_layout)
        lc.reserve((size_t)C0);
        int32_t cs = 0;
        for (int a = 0; a < m; ++a) {
          const int32_t nc = (int32_t)ceil_div(sh.h_col_len[a], kChunk);
          if (!flag[(size_t)a])
            for (int32_t k = 0; k < nc; ++k) lc.push_back(cs + k);
          cs += nc;
        }
        const int32_t nlc = (int32_t)lc.size();
        // warp batches: 32/W lists of root length <= W (W a power of two), longest first
        std::vector<int2> batch;
        for (size_t i = 0; i < attrs.size();) {
          const int64_t L = sh.h_col_len[(size_t)attrs[i]];
          int lw = 0;
          while ((1 << lw) < L) ++lw;
          const int cnt = (int)std::min<size_t>((size_t)(32 >> lw), attrs.size() - i);
          batch.push_back(make_int2((int)i, cnt | (lw << 16)));
          i += (size_t)cnt;
        }
        Carve zp{nullptr};
        auto zs = [&](Carve& z) {
          z.take<int32_t>(attrs.size()); z.take<uint8_t>((size_t)m); z.take<int32_t>((size_t)C0); z.take<int32_t>(4);
          z.take<int32_t>((size_t)C0); z.take<int32_t>((size_t)C0); z.take<int2>(batch.size());
          z.take<uint8_t>((size_t)sh.cap); z.take<uint8_t>((size_t)sh.cap); z.take<int32_t>(longa.size() + 1);
        };
        zs(zp);
        w.shortmem.alloc(zp.off + 1024, st);
        Carve z{w.shortmem.as<char>()};
        int32_t* d_attrs = z.take<int32_t>(attrs.size());
        w.sflag = z.take<uint8_t>((size_t)m);
        int32_t* rlc = z.take<int32_t>((size_t)C0);
        int32_t* nl = z.take<int32_t>(4);
        w.tab[0].lc = z.take<int32_t>((size_t)C0);
        w.tab[1].lc = z.take<int32_t>((size_t)C0);
        int2* d_batch = z.take<int2>(batch.size());
        w.jl[0] = z.take<uint8_t>((size_t)sh.cap);
        w.jl[1] = z.take<uint8_t>((size_t)sh.cap);
        w.longa = z.take<int32_t>(longa.size() + 1);
        w.nlong = (int)longa.size();
        if (!longa.empty())
          GBDT_CUDA(cudaMemcpyAsync(w.longa, longa.data(), 4 * longa.size(), cudaMemcpyHostToDevice, st));
        w.root.lc = rlc;
        w.root.nlc = nl;
        w.tab[0].nlc = nl + 1;
        w.tab[1].nlc = nl + 2;
        GBDT_CUDA(cudaMemcpyAsync(d_attrs, attrs.data(), 4 * attrs.size(), cudaMemcpyHostToDevice, st));
        GBDT_CUDA(cudaMemcpyAsync(w.sflag, flag.data(), (size_t)m, cudaMemcpyHostToDevice, st));
        if (nlc) GBDT_CUDA(cudaMemcpyAsync(rlc, lc.data(), 4 * (size_t)nlc, cudaMemcpyHostToDevice, st));
        GBDT_CUDA(cudaMemcpyAsync(nl, &nlc, 4, cudaMemcpyHostToDevice, st));
        GBDT_CUDA(cudaMemcpyAsync(d_batch, batch.data(), sizeof(int2) * batch.size(), cudaMemcpyHostToDevice, st));
        GBDT_CUDA(cudaStreamSynchronize(st));  // the host vectors must outlive the copies
        w.sl.attrs = d_attrs;
        w.sl.n = (int)attrs.size();
        w.sl.batch = d_batch;
        w.sl.nb = (int)batch.size();
        // in-place short lists when every level of the tree is on the short path (depth <= 6):
        // no partition of them at all (GBDT_SHORT_INPLACE=0: partitioned like the other lists)
        bool inplace = d <= kShortLevels && cap_level < 0 && !sh.rle;
        if (const char* e = getenv("GBDT_SHORT_INPLACE")) inplace = inplace && e[0] != '0';
        if (inplace) {
          w.shortg.alloc((size_t)sh.cap * 8 * (hmode == kHGather ? 2 : 1) + 64, st);
          w.sl.inplace = 1;
          w.sl.cs0 = w.root.col_start;
          w.sl.cl0 = w.root.col_len;
          w.sl.val0 = sh.val0.as<float>();
          w.sl.ins0 = sh.ins0.as<int32_t>();
          w.sl.gsh = w.shortg.as<double>();
          w.sl.hsh = hmode == kHGather ? w.shortg.as<double>() + sh.cap : nullptr;
        }
      }
    }
    w.nrec = nrec + li;
    w.gkey = gkey + (size_t)li * Kcap;
    w.tkey = tkey + (size_t)li * Kcap;
  }

  PhaseTimer tm, kt;  // phases; kernel-level timers nested inside them
  tm.on = kt.on = P.profile != 0;
  tm.nvtx = true;
  tm.st = kt.st = st;
  cudaEvent_t tot0 = nullptr, tot1 = nullptr;
  if (tm.on) {
    GBDT_CUDA(cudaEventCreate(&tot0));
    GBDT_CUDA(cudaEventCreate(&tot1));
    GBDT_CUDA(cudaEventRecord(tot0, st));
  }
  const double thr = P.gamma > 0 ? P.gamma : 0.0;

  // Several local shards: their partitions and next-level split finds run pipelined on one stream
  // each (profiling, the fused pass and the level-capture hook keep the sequential order;
  // GBDT_PIPE=0 forces it)
  bool pipe = nloc > 1 && !tm.on && !fused && cap_level < 0 && !custom;
  if (const char* pe = getenv("GBDT_PIPE")) pipe = pipe && pe[0] != '0';
  struct PipeRes {
    std::vector<cudaStream_t> st;
    std::vector<cudaEvent_t> ev;
    ~PipeRes() {
      for (auto e : ev) cudaEventDestroy(e);
      for (auto x : st) cudaStreamDestroy(x);
    }
  } pres;
  if (pipe) {
    pres.st.resize(nloc, nullptr);
    pres.ev.resize(1 + 2 * (size_t)nloc, nullptr);
    for (auto& x : pres.st) GBDT_CUDA(cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking));
    for (auto& e : pres.ev) GBDT_CUDA(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
  }
  cudaStream_t* pst = pres.st.data();
  cudaEvent_t* pev = pres.ev.data();

  // One tree of Alg. 1 (every tree-dependent pointer is resolved on the device from tidx, so the
  // same launch sequence builds any tree): captured once into a CUDA graph and replayed T times
  // when nothing in it needs the host (no profiling events, no user-loss callback, no
  // host-staged collectives); launched directly otherwise.
  auto tree_body = [&](int t) {
    nvtxRangePushA("tree");
    tm.begin(GBDT_PHASE_GRAD);
    if (rows.indptr) rows.trees = trees;
    k_grad<<<grad_blocks, 256, 0, st>>>(n, P.loss, tidx, P.eta, P.base_margin, ds.y.as<float>(), hweight, NH,
                                        yhat, pos, gv, hv, hmode == kHGather, partial, rows, custom ? 1 : 0, tidx + 2);
    GBDT_LAUNCH_CHECK();
    if (custom) {  // user-defined loss: g, h from the callback, on this stream
      if (P.grad_fn(n, yhat, ds.y.as<float>(), gv, hv, (void*)st, P.grad_user) != 0)
        fail(GBDT_E_INVAL, "grad_fn failed at tree " + std::to_string(t));
      GBDT_CUDA(cudaMemsetAsync(tidx + 2, 0, sizeof(int32_t), st));
      k_grad<<<grad_blocks, 256, 0, st>>>(n, P.loss, tidx, P.eta, P.base_margin, ds.y.as<float>(), hweight, NH,
                                          yhat, pos, gv, hv, 1, partial, RowsArgs{}, 2, tidx + 2);
      GBDT_LAUNCH_CHECK();
      count_launch();
      int32_t bad = 0;  // the custom path runs eagerly: check the callback's g, h before using them
      GBDT_CUDA(cudaMemcpyAsync(&bad, tidx + 2, sizeof bad, cudaMemcpyDeviceToHost, st));
      GBDT_CUDA(cudaStreamSynchronize(st));
      if (bad) fail(GBDT_E_INVAL, "grad_fn returned a non-finite g or h, or h < 0, at tree " + std::to_string(t));
    }
    k_tree_begin<<<1, 1024, 0, st>>>(grad_blocks, partial, n, P.lambda, nt[0], NH, hweight, hstate, trees, fxs, tidx,
                                     tloss);
    GBDT_LAUNCH_CHECK();
    count_launch(2);
    tm.end();

    // split find of level L for local shard li on stream s (a3-a6)
    auto split_shard = [&](int li, int L, cudaStream_t s) {
      const int lvl = L;
      NodeTab& cur = nt[L & 1];
      cudaStream_t st = s;
        Shard& sh = *ds.shards[li];
        ShardWork& w = sw[li];
        if (sh.m == 0) return;
        const Tables tb = lvl == 0 ? w.root : w.tab[lvl & 1];
        const float* val = lvl == 0 ? sh.val0.as<float>() : sh.valw[lvl & 1].as<float>();
        const int32_t* ins = lvl == 0 ? sh.ins0.as<int32_t>() : sh.insw[lvl & 1].as<int32_t>();
        SplitArgs A;
        A.t = TileArgs{val, ins, tb, sh.m, sh.a_begin, cur.K, w.counters, w.level_flag(lvl)};
        A.desc = w.desc; A.rle = sh.rle ? 1 : 0; A.genlist = w.genlist; A.ngen = w.counters + 2;
        A.g = gv; A.h = hv; A.nodes = cur; A.segPG = w.segPG; A.segPH = w.segPH; A.lam = P.lambda;
        A.epochp = epoch; A.fx = fxs; A.rec = w.rec;
        A.glist = w.glist[lvl & 1]; A.hlist = w.hlist[lvl & 1]; A.cagg = w.cagg; A.carry = w.carry;
        A.sgrp = w.sgrp; A.nrec = w.nrec; A.gkey = w.gkey; A.shard = sh.index;
        A.segPG_out = w.segPG; A.segPH_out = w.segPH;
        // present totals per segment (needed for the missing direction), from the chunk pass
        A.segEnd = ds.has_missing ? w.segEnd : nullptr;
        if (w.level_flag(lvl)) { A.longa = w.longa; A.nlong = w.nlong; }
        const bool rs = runsplit && sh.rle;
        kt.begin(GBDT_PHASE_K_CHUNK_AGG);
        if (rs) {
          // the split on runs gathers the root g-list itself (k_run_root)
        } else if (lvl > 0 && !ds.has_missing) {
          LK.chunk_desc(A, w.groups, st);  // aggregates from the scatter
        } else {
          LK.tile_prefix(A, hmode, /*gather=*/lvl == 0, w.groups, st);
        }
        kt.end();

        kt.begin(GBDT_PHASE_K_SPLIT);
        if (rs) {
          LK.run_split(A, hmode, /*root=*/lvl == 0, w.racc, w.rcar, w.rsg5, w.rgroups, st);
        } else {
          LK.short_split(A, w.level_sl(lvl), hmode, /*gather=*/lvl == 0, st);
          LK.split_find(A, hmode, ds.has_missing, sh.rle, st);
        }
        kt.end();
        if (P.profile) {  // the level's list entries (byte model of the bench), off the timed kernels
          k_level_entries<<<(unsigned)std::min<int64_t>(ceil_div(sh.m, 256), sms * 4), 256, 0, st>>>(tb.col_len, sh.m, lent + lvl);
          GBDT_LAUNCH_CHECK();
          count_launch();
        }
    };
    // partition of level L for local shard li on stream s (a8); ev_count: recorded after the count
    auto part_shard = [&](int li, int L, cudaStream_t s, cudaEvent_t ev_count) {
      const int lvl = L;
      NodeTab& cur = nt[L & 1];
      NodeTab& nxt = nt[(L + 1) & 1];
      const int Kl = 1 << L;
      cudaStream_t st = s;
      (void)cur;
        Shard& sh = *ds.shards[li];
        ShardWork& w = sw[li];
        if (sh.m == 0) return;
        const Tables tb = lvl == 0 ? w.root : w.tab[lvl & 1];
        const Tables tn = w.tab[(lvl + 1) & 1];
        const float* val = lvl == 0 ? sh.val0.as<float>() : sh.valw[lvl & 1].as<float>();
        const int32_t* ins = lvl == 0 ? sh.ins0.as<int32_t>() : sh.insw[lvl & 1].as<int32_t>();
        if (ds.has_missing) {
          const size_t Sl = (size_t)sh.m * Kl;
          GBDT_CUDA(cudaMemsetAsync(w.segH, 0, Sl * 4, st));
          GBDT_CUDA(cudaMemsetAsync(w.segL, 0, Sl * 4, st));
        }
        PartArgs PA;
        PA.t = TileArgs{val, ins, tb, sh.m, sh.a_begin, cur.K, w.counters + 1, w.level_flag(lvl)};
        const ShortList lsl = w.level_sl(lvl);
        PA.side = side; PA.hbit = hbit; PA.cidx = cidx; PA.slist = w.slist; PA.segH = w.segH; PA.segL = w.segL;
        PA.seg_pre = w.seg_pre; PA.out_hi = w.out_hi; PA.out_lo = w.out_lo;
        PA.val_out = sh.valw[(lvl + 1) & 1].as<float>();
        PA.ins_out = sh.insw[(lvl + 1) & 1].as<int32_t>();
        PA.ccnt = w.ccnt; PA.cpre = w.cpre; PA.sgrp = w.sgrp;
        PA.g_in = w.glist[lvl & 1]; PA.h_in = w.hlist[lvl & 1];
        PA.g_out = w.glist[(lvl + 1) & 1]; PA.h_out = w.hlist[(lvl + 1) & 1];
        PA.epochp = epoch;
        // without missing values the scatter accumulates the next level's chunk aggregates
        PA.cagg_next = (ds.has_missing || (runsplit && sh.rle)) ? nullptr : w.cagg;
        PA.nxt = tn;
        PA.fx = fxs;
        PlanArgs PL;
        PL.m = sh.m; PL.counted = ds.has_missing; PL.Kp = cur.K; PL.Knp = nxt.K; PL.cidx = cidx; PL.ncnt = nxt.cnt;
        PL.segH = w.segH; PL.segL = w.segL; PL.seg_pre = w.seg_pre;
        PL.out_hi = w.out_hi; PL.out_lo = w.out_lo; PL.len_tmp = w.len_tmp; PL.nxt = tn;
        PL.el = w.pel; PL.egrp = w.pgrp; PL.egroups = w.pgroups; PL.mp1 = w.mp1; PL.sflag = w.level_flag(lvl + 1);
        PL.inplace = w.sl.inplace;
        RunArgs RA;
        if (sh.rle) {
          RA.m = sh.m; RA.Kp = cur.K; RA.Knp = nxt.K; RA.cidx = cidx; RA.cur = tb; RA.nxt = tn;
          RA.slist = w.slist; RA.cpre = w.cpre; RA.run_seg = w.run_seg; RA.run_hl = w.run_hl; RA.cnt = w.rcnt; RA.fl = w.rfl;
          RA.Rp1 = w.Rp1; RA.sgrp = w.rsgrp; RA.groups = w.rgroups;
        }
        // RLE split ablation (gbdt_params.rle_decompress, Fig. 6): the runs are decompressed
        // into the level's value list, the lists partitioned as plain ones, the children re-encoded
        const bool dec = sh.rle && P.rle_decompress;
        if (dec && lvl > 0) {
          LK.rle_decompress(tb, sh.valw[lvl & 1].as<float>(), st);
          PA.t.val = sh.valw[lvl & 1].as<float>();
        }
        kt.begin(GBDT_PHASE_K_COUNT);
        LK.partition_count(PA, PL, ds.has_missing, w.groups, st, &lsl);
        if (ev_count) GBDT_CUDA(cudaEventRecord(ev_count, st));  // the next shard's count may start
        kt.end();
        kt.begin(GBDT_PHASE_K_SCATTER);
        if (PA.cagg_next)
          GBDT_CUDA(cudaMemsetAsync(w.cagg, 0, sizeof(unsigned long long) * 5 * (size_t)std::max<int64_t>(sh.C0, 1), st));
        LK.partition_scatter(PA, hmode, (sh.rle && !dec) ? &RA : nullptr, st, &lsl);
        if (dec)
          LK.rle_encode(tn, sh.m, nxt.K, sh.valw[(lvl + 1) & 1].as<float>(), w.enc_cnt, w.enc_bits,
                        ((size_t)sh.cap / 32 + 2) * 4, st);
        kt.end();
    };
    for (int lvl = 0; lvl < d; ++lvl) {
      NodeTab& cur = nt[lvl & 1];
      NodeTab& nxt = nt[(lvl + 1) & 1];
      const bool last = (lvl == d - 1);
      const int Kl = 1 << lvl;  // upper bound of active nodes at this level
      if (cap_level == lvl && t == 0) {  // test hook: this level's lists and tables, tree 0
        GBDT_CUDA(cudaStreamSynchronize(st));
        int32_t Kh = 0;
        GBDT_CUDA(cudaMemcpy(&Kh, cur.K, 4, cudaMemcpyDeviceToHost));
        model.captures.clear();
        for (int li = 0; li < nloc; ++li) {
          Shard& sh = *ds.shards[li];
          const Tables tb = lvl == 0 ? sw[li].root : sw[li].tab[lvl & 1];
          LevelCapture L;
          L.shard = sh.index;
          L.K = Kh;
          L.col_start.resize((size_t)sh.m + 1);
          L.col_len.resize((size_t)sh.m);
          L.seg_start.resize((size_t)sh.m * Kh);
          L.seg_cnt.resize((size_t)sh.m * Kh);
          if (sh.m) {
            GBDT_CUDA(cudaMemcpy(L.col_start.data(), tb.col_start, 8 * ((size_t)sh.m + 1), cudaMemcpyDeviceToHost));
            GBDT_CUDA(cudaMemcpy(L.col_len.data(), tb.col_len, 8 * (size_t)sh.m, cudaMemcpyDeviceToHost));
            GBDT_CUDA(cudaMemcpy(L.seg_start.data(), tb.seg_start, 8 * L.seg_start.size(), cudaMemcpyDeviceToHost));
            GBDT_CUDA(cudaMemcpy(L.seg_cnt.data(), tb.seg_cnt, 8 * L.seg_cnt.size(), cudaMemcpyDeviceToHost));
          }
          const size_t len = (size_t)L.col_start[sh.m];
          L.val.resize(len);
          L.ins.resize(len);
          const float* val = lvl == 0 ? sh.val0.as<float>() : sh.valw[lvl & 1].as<float>();
          const int32_t* ins = lvl == 0 ? sh.ins0.as<int32_t>() : sh.insw[lvl & 1].as<int32_t>();
          if (len) {
            GBDT_CUDA(cudaMemcpy(L.val.data(), val, 4 * len, cudaMemcpyDeviceToHost));
            GBDT_CUDA(cudaMemcpy(L.ins.data(), ins, 4 * len, cudaMemcpyDeviceToHost));
          }
          if (sh.rle) {
            int32_t R = 0;
            GBDT_CUDA(cudaMemcpy(&R, tb.R, 4, cudaMemcpyDeviceToHost));
            L.seg_run.resize((size_t)sh.m * Kh + 1);
            L.run_val.resize((size_t)R);
            L.run_len.resize((size_t)R);
            L.run_pos.resize((size_t)R);
            GBDT_CUDA(cudaMemcpy(L.seg_run.data(), tb.seg_run, 4 * L.seg_run.size(), cudaMemcpyDeviceToHost));
            if (R) {
              GBDT_CUDA(cudaMemcpy(L.run_val.data(), tb.run_val, 4 * (size_t)R, cudaMemcpyDeviceToHost));
              GBDT_CUDA(cudaMemcpy(L.run_len.data(), tb.run_len, 4 * (size_t)R, cudaMemcpyDeviceToHost));
              GBDT_CUDA(cudaMemcpy(L.run_pos.data(), tb.run_pos, 8 * (size_t)R, cudaMemcpyDeviceToHost));
            }
          }
          model.captures.push_back(std::move(L));
        }
      }
      // fz: this level's node bests were found by the previous level's fused pass
      const bool fz = fused && lvl >= 1;
      if (!fz && !(pipe && lvl > 0)) {
      tm.begin(GBDT_PHASE_DECIDE);
      k_level_begin<<<1, 1024, 0, st>>>(epoch, sw[0].counters, 0, nrec, nloc, cur.K, gkey, tkey, Kcap);
      GBDT_LAUNCH_CHECK();
      count_launch();
      for (int li = 0; li < nloc; ++li) GBDT_CUDA(cudaMemsetAsync(sw[li].counters, 0, 4 * sizeof(int), st));
      tm.end();
      }
      tm.begin(GBDT_PHASE_SPLIT_FIND);
      for (int li = 0; li < nloc && !fz; ++li) {
        if (pipe && lvl > 0) break;  // found by the pipelined partition of the previous level
        split_shard(li, lvl, st);
      }
      tm.end();
      tm.begin(GBDT_PHASE_DECIDE);
      for (int li = 0; li < nloc; ++li) {
        ShardWork& w = sw[li];
        Rec* bo = best_all + (size_t)ds.shards[li]->index * Kcap;
        k_pick_tie<<<sms * 2, 256, 0, st>>>(w.rec, w.nrec, w.gkey, w.tkey);
        k_pick_best<<<sms * 2, 256, 0, st>>>(w.rec, w.nrec, w.gkey, w.tkey, bo);
        GBDT_LAUNCH_CHECK();
        count_launch(2);
      }
      tm.end();
      if (ds.comm) {  // every rank (a world of 1 too: the same calls, trivially)
        tm.begin(GBDT_PHASE_COMM);
        Rec* mine = best_all + (size_t)ds.shards[0]->index * Kcap;
        ds.comm->allgather(mine, best_all, sizeof(Rec) * Kcap, st);
        tm.end();
      }
      tm.begin(GBDT_PHASE_DECIDE);
      DecideArgs D;
      D.cur = cur; D.nxt = nxt; D.best_all = best_all; D.nshard = nsh; D.Kcap = Kcap; D.epochp = epoch;
      D.lam = P.lambda; D.thr = thr; D.last_level = last; D.cidx = cidx; D.winner = winner;
      D.hstate = hstate; D.hdef = hdef; D.hweight = hweight; D.trees = trees; D.tidx = tidx; D.NH = NH;
      k_decide<<<1, 1024, 0, st>>>(D);
      GBDT_LAUNCH_CHECK();
      count_launch();
      tm.end();

      tm.begin(GBDT_PHASE_NODEMAP);
      const size_t bit_bytes = ((size_t)n + 31) / 32 * 4;
      GBDT_CUDA(cudaMemsetAsync(bits, 0, bit_bytes, st));
      for (int li = 0; li < nloc; ++li) {
        Shard& sh = *ds.shards[li];
        if (sh.m == 0) continue;
        if (fz) {  // the winners' child segments, read from the parent level's lists
          const int32_t* pins = lvl == 1 ? sh.ins0.as<int32_t>() : sh.insw[(lvl - 1) & 1].as<int32_t>();
          fused_mark(sw[li].fplan[(lvl - 1) & 1], cur.K, cidx, winner, sh.index, sh.a_begin, pins,
                     hbitF[(lvl - 1) & 1], bits, n, Kl, sms, st);
          continue;
        }
        const Tables tb = lvl == 0 ? sw[li].root : sw[li].tab[lvl & 1];
        const int32_t* ins = lvl == 0 ? sh.ins0.as<int32_t>() : sh.insw[lvl & 1].as<int32_t>();
        dim3 grid((unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256 * (int64_t)Kl), (int64_t)sms * 4)), (unsigned)Kl);
        k_mark<<<grid, 256, 0, st>>>(cur.K, cidx, winner, sh.index, sh.a_begin, tb, ins, bits,
                                     sw[li].level_flag(lvl), sw[li].level_sl(lvl));
        GBDT_LAUNCH_CHECK();
        count_launch();
      }
      tm.end();
      if (ds.comm) {
        tm.begin(GBDT_PHASE_COMM);
        // the ranks' bits are disjoint (one owner shard per node), so a byte-wise sum is their OR:
        // n/8 bytes on the wire (1.4 MB for C3)
        ds.comm->allreduce_sum_u8(bits, bit_bytes, st);
        tm.end();
      }
      tm.begin(GBDT_PHASE_NODEMAP);
      k_nodemap<<<inst_grid, 256, 0, st>>>(n, bits, hstate, hdef, pos, side, fused ? hbitF[lvl & 1] : hbit);
      GBDT_LAUNCH_CHECK();
      count_launch();
      tm.end();

      if (last) break;
      tm.begin(GBDT_PHASE_PARTITION);
      if (fused) {  // partition of this level + split find of the next, one pass (fused.cu)
        k_level_begin<<<1, 1024, 0, st>>>(epoch, sw[0].counters, 0, nrec, nloc, nxt.K, gkey, tkey, Kcap);
        GBDT_LAUNCH_CHECK();
        count_launch();
        for (int li = 0; li < nloc; ++li) {
          Shard& sh = *ds.shards[li];
          ShardWork& w = sw[li];
          if (sh.m == 0) continue;
          FusedArgs FA;
          fused_carve(FA, w.tilemem, w.tiles);
          fused_plan(w.fplan[lvl & 1], cur, nxt, cidx, epoch, sh.m, P.profile ? lent : nullptr, lvl, FA.mcount, st);
          FA.val = lvl == 0 ? sh.val0.as<float>() : sh.valw[lvl & 1].as<float>();
          FA.ins = lvl == 0 ? sh.ins0.as<int32_t>() : sh.insw[lvl & 1].as<int32_t>();
          FA.gl = w.glist[lvl & 1];
          FA.val_out = sh.valw[(lvl + 1) & 1].as<float>();
          FA.ins_out = sh.insw[(lvl + 1) & 1].as<int32_t>();
          FA.g_out = w.glist[(lvl + 1) & 1];
          FA.hbit = hbitF[lvl & 1];
          FA.plan = w.fplan[lvl & 1];
          FA.nxt = nxt;
          {
            const char* fw = getenv("GBDT_FUSEDW");
            FA.warp_tiles = fw ? fw[0] != '0' : 1;
          }
          FA.fx = fxs; FA.lam = P.lambda; FA.m = sh.m; FA.a_base = sh.a_begin; FA.shard = sh.index;
          FA.rec = w.rec; FA.nrec = w.nrec; FA.gkey = w.gkey;
          kt.begin(GBDT_PHASE_K_FUSED);
          fused_pass(FA, hmode, /*write=*/lvl + 1 < d - 1, w.tiles, st);
          kt.end();
        }
        tm.end();
        continue;
      }
      if (pipe) {
        // Pipelined over the local shards (one stream each): shard li's partition of this level
        // and its split find of the next; its count starts when shard li-1's count is done, so
        // the L1TEX-bound count of one shard overlaps the DRAM-bound scatter and the issue-bound
        // split find of the others.  The next level's begin runs first, on st.
        k_level_begin<<<1, 1024, 0, st>>>(epoch, sw[0].counters, 0, nrec, nloc, nxt.K, gkey, tkey, Kcap);
        GBDT_LAUNCH_CHECK();
        count_launch();
        for (int li = 0; li < nloc; ++li) GBDT_CUDA(cudaMemsetAsync(sw[li].counters, 0, 4 * sizeof(int), st));
        GBDT_CUDA(cudaEventRecord(pev[0], st));
        for (int li = 0; li < nloc; ++li) {
          cudaStream_t ss = pst[li];
          GBDT_CUDA(cudaStreamWaitEvent(ss, pev[0], 0));
          if (li > 0) GBDT_CUDA(cudaStreamWaitEvent(ss, pev[1 + (li - 1)], 0));
          part_shard(li, lvl, ss, pev[1 + li]);
          split_shard(li, lvl + 1, ss);
          GBDT_CUDA(cudaEventRecord(pev[1 + nloc + li], ss));
        }
        for (int li = 0; li < nloc; ++li) GBDT_CUDA(cudaStreamWaitEvent(st, pev[1 + nloc + li], 0));
      } else {
        for (int li = 0; li < nloc; ++li) part_shard(li, lvl, st, nullptr);
      }
      tm.end();
    }
    k_tree_end<<<1, 1, 0, st>>>(tidx);
    GBDT_LAUNCH_CHECK();
    count_launch();
    nvtxRangePop();
  };

  // One CUDA graph per tree, NCCL collectives included (captured on the library's stream; a world
  // of one rank exercises the same captured calls on single-GPU boxes).  GBDT_GRAPH=0 forces eager
  // launches.  Host-staged collectives (callbacks) cannot be captured.
  const bool host_comm = ds.comm && !ds.comm->nccl;
  const char* ge = getenv("GBDT_GRAPH");
  const bool graph_ok = ge ? ge[0] != '0' : true;
  const bool graph = !tm.on && !custom && !host_comm && P.n_trees > 1 && graph_ok && cap_level < 0;
  if (!graph) {
    for (int t = 0; t < P.n_trees; ++t) tree_body(t);
  } else {
    // capture on a private stream (the legacy default stream cannot be captured); nothing runs
    // during the capture, the replays go to st in order
    const cudaStream_t st0 = st;
    cudaStream_t cs = nullptr;
    GBDT_CUDA(cudaStreamCreateWithFlags(&cs, cudaStreamNonBlocking));
    cudaGraph_t g = nullptr;
    cudaGraphExec_t gx = nullptr;
    const int64_t before = launches_get();
    st = cs;
    GBDT_CUDA(cudaStreamBeginCapture(cs, cudaStreamCaptureModeThreadLocal));
    try {
      tree_body(0);
    } catch (...) {
      cudaStreamEndCapture(cs, &g);
      if (g) cudaGraphDestroy(g);
      st = st0;
      cudaStreamDestroy(cs);
      throw;
    }
    GBDT_CUDA(cudaStreamEndCapture(cs, &g));
    st = st0;
    const int64_t per_tree = launches_get() - before;
    launches_reset();
    count_launch((int)before);
    GBDT_CUDA(cudaGraphInstantiate(&gx, g, 0));
    for (int t = 0; t < P.n_trees; ++t) {
      GBDT_CUDA(cudaGraphLaunch(gx, st));
      count_launch((int)per_tree);
    }
    GBDT_CUDA(cudaGraphExecDestroy(gx));
    GBDT_CUDA(cudaGraphDestroy(g));
    GBDT_CUDA(cudaStreamDestroy(cs));
  }
  // final SmartGD step: the last tree's leaf weights
  {
    double* wlast = hweight + (size_t)((P.n_trees - 1) & 1) * NH;
    if (rows.indptr) {  // ablation: the final margin by traversal of all trees too
      rows.trees = trees; rows.t = P.n_trees;
      k_grad<<<grad_blocks, 256, 0, st>>>(n, P.loss, nullptr, P.eta, P.base_margin, ds.y.as<float>(), hweight, NH,
                                          yhat, pos, gv, hv, 0, partial, rows, 1, tidx + 2);
    } else {
      k_apply<<<inst_grid, 256, 0, st>>>(n, P.eta, wlast, pos, yhat);
    }
    GBDT_LAUNCH_CHECK();
    count_launch();
    k_loss_partial<<<grad_blocks, 256, 0, st>>>(n, P.loss, yhat, ds.y.as<float>(), partial);
    k_loss_final<<<1, 1, 0, st>>>(grad_blocks, partial, n, custom ? 1 : 0, tloss + P.n_trees);
    GBDT_LAUNCH_CHECK();
    count_launch(2);
  }
  if (tm.on) GBDT_CUDA(cudaEventRecord(tot1, st));
  model.n_trees = P.n_trees;
  model.max_depth = d;
  model.loss = P.loss;
  model.n_cols = ds.m;
  model.eta = P.eta;
  model.base_margin = P.base_margin;
  model.dense = ds.dense;
  model.fill = ds.fill;
  model.lambda = P.lambda;
  model.device = ds.device;
  model.nodes.resize((size_t)P.n_trees * NH);
  model.level_entries.assign(d, 0);
  if (P.profile) {
    std::vector<unsigned long long> le(16, 0);
    GBDT_CUDA(cudaMemcpyAsync(le.data(), lent, sizeof(unsigned long long) * 16, cudaMemcpyDeviceToHost, st));
    GBDT_CUDA(cudaStreamSynchronize(st));
    for (int l = 0; l < d && l < 16; ++l) model.level_entries[l] = (int64_t)le[l];
  }
  GBDT_CUDA(cudaMemcpyAsync(model.nodes.data(), trees, sizeof(gbdt_node) * model.nodes.size(),
                            cudaMemcpyDeviceToHost, st));
  model.train_loss.assign((size_t)P.n_trees + 1, 0.0);
  GBDT_CUDA(cudaMemcpyAsync(model.train_loss.data(), tloss, sizeof(double) * (P.n_trees + 1), cudaMemcpyDeviceToHost, st));
  if (margin_out)
    GBDT_CUDA(cudaMemcpyAsync(margin_out, yhat, sizeof(double) * (size_t)n, cudaMemcpyDeviceToHost, st));
  GBDT_CUDA(cudaStreamSynchronize(st));
  for (int i = 0; i < GBDT_N_PHASES; ++i) model.timings[i] = 0.0;
  if (tm.on) {
    tm.collect(model.timings);
    kt.collect(model.timings);
    float tt = 0;
    GBDT_CUDA(cudaEventElapsedTime(&tt, tot0, tot1));
    model.timings[GBDT_PHASE_TOTAL] = tt;
    cudaEventDestroy(tot0);
    cudaEventDestroy(tot1);
  }
}

}  // namespace gbdt
