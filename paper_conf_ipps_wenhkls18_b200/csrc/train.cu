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
// Determinism: all fp64 sums use fixed association.  The cross-tile carry of the segmented scan
// is a Fenwick tree over the tiles of ONE attribute (tiles are attribute-aligned), so every
// attribute's prefix sums -- hence its gains -- are bit-identical whatever else is in the level
// buffer (other attributes, other shards, other runs).  The per-node argmax is over a strict
// total order (gain desc, attr asc, value desc, dir), so its result does not depend on the order
// in which pieces are reduced.
#include <algorithm>
#include <cstring>
#include <vector>

#include "kernels.cuh"

namespace gbdt {

namespace {

thread_local int64_t g_launches = 0;

// ============================================================================ scan helpers
struct SVf {
  double g, h;
  int c, f;
};
__device__ __forceinline__ SVf svf_zero() { return SVf{0.0, 0.0, 0, 0}; }
// segmented combine: a head in the right operand discards the left one
__device__ __forceinline__ SVf comb(const SVf& l, const SVf& r) {
  if (r.f) return r;
  return SVf{l.g + r.g, l.h + r.h, l.c + r.c, l.f};
}
__device__ __forceinline__ SVf shfl_up(const SVf& x, int o) {
  SVf y;
  y.g = __shfl_up_sync(0xffffffffu, x.g, o);
  y.h = __shfl_up_sync(0xffffffffu, x.h, o);
  y.c = __shfl_up_sync(0xffffffffu, x.c, o);
  y.f = __shfl_up_sync(0xffffffffu, x.f, o);
  return y;
}
__device__ __forceinline__ SVf shfl_idx(const SVf& x, int l) {
  SVf y;
  y.g = __shfl_sync(0xffffffffu, x.g, l);
  y.h = __shfl_sync(0xffffffffu, x.h, l);
  y.c = __shfl_sync(0xffffffffu, x.c, l);
  y.f = __shfl_sync(0xffffffffu, x.f, l);
  return y;
}

// argmax element within a piece (attr fixed): gain desc, value desc, dir low first (R12)
struct AM {
  double gain;
  float value;
  int meta;  // bits 0-11 item index in tile, bit 12 dir, bit 13 valid
  int f;     // piece start inside
};
__device__ __forceinline__ AM am_none() { return AM{0.0, 0.f, 0, 0}; }
__device__ __forceinline__ bool am_valid(const AM& a) { return (a.meta >> 13) & 1; }
__device__ __forceinline__ AM am_best(const AM& a, const AM& b) {
  if (!am_valid(a)) return b;
  if (!am_valid(b)) return a;
  if (a.gain != b.gain) return a.gain > b.gain ? a : b;
  if (a.value != b.value) return a.value > b.value ? a : b;
  return ((a.meta >> 12) & 1) <= ((b.meta >> 12) & 1) ? a : b;
}
__device__ __forceinline__ AM am_comb(const AM& l, const AM& r) {
  if (r.f) return r;
  AM x = am_best(l, r);
  x.f = l.f;
  return x;
}
__device__ __forceinline__ AM shfl_up(const AM& x, int o) {
  AM y;
  y.gain = __shfl_up_sync(0xffffffffu, x.gain, o);
  y.value = __shfl_up_sync(0xffffffffu, x.value, o);
  y.meta = __shfl_up_sync(0xffffffffu, x.meta, o);
  y.f = __shfl_up_sync(0xffffffffu, x.f, o);
  return y;
}

// ============================================================================ tile metadata
struct TileMeta {
  long long p0, p1, colend;
  long long sb;  // first segment index of the attribute (a*K)
  int t, a, u, j0, jlast;
};

// Thread 0 only.  Tiles never straddle attributes (attribute-aligned tiling).
__device__ void tile_meta(const TileArgs& A, int K, int t, TileMeta& M) {
  int lo = 0, hi = A.m - 1;  // largest a with tile_start[a] <= t
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (A.tb.tile_start[mid] <= t) lo = mid; else hi = mid - 1;
  }
  const int a = lo;
  M.t = t;
  M.a = a;
  M.u = t - A.tb.tile_start[a];
  const long long cs = A.tb.col_start[a];
  M.colend = cs + A.tb.col_len[a];
  M.p0 = cs + (long long)M.u * kTile;
  M.p1 = min(M.p0 + (long long)kTile, M.colend);
  M.sb = (long long)a * K;
  const int64_t* ss = A.tb.seg_start + M.sb;
  lo = 0; hi = K - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (ss[mid] <= M.p0) lo = mid; else hi = mid - 1;
  }
  M.j0 = lo;
  hi = K - 1;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (ss[mid] <= M.p1 - 1) lo = mid; else hi = mid - 1;
  }
  M.jlast = lo;
}

// Assigns each of the thread's items to its (node) segment; sets head / piece-end / run-end masks.
template <bool kNeedVal>
__device__ __forceinline__ void assign_segments(const TileArgs& A, const TileMeta& M, long long base,
                                                unsigned vm, const float* v, float vnext, int* sj,
                                                unsigned& hm, unsigned& pem, unsigned& rem) {
  hm = pem = rem = 0;
  if (!vm) return;
  const int64_t* ss = A.tb.seg_start + M.sb;
  const int64_t* sc = A.tb.seg_cnt + M.sb;
  int lo = M.j0, hi = M.jlast;
  while (lo < hi) {
    int mid = (lo + hi + 1) >> 1;
    if (ss[mid] <= base) lo = mid; else hi = mid - 1;
  }
  int j = lo;
  long long s0 = ss[j], se = s0 + sc[j];
#pragma unroll
  for (int k = 0; k < kItems; ++k) {
    const long long p = base + k;
    if (!((vm >> k) & 1)) { sj[k] = j; continue; }
    while (p >= se) { ++j; s0 = ss[j]; se = s0 + sc[j]; }
    sj[k] = j;
    if (p == s0) hm |= 1u << k;
    const bool seg_last = (p + 1 == se);
    if (seg_last || p + 1 == M.p1) pem |= 1u << k;
    if (kNeedVal) {
      const float nv = (k < kItems - 1) ? v[k + 1] : vnext;
      if (seg_last || nv != v[k]) rem |= 1u << k;
    } else if (seg_last) {
      rem |= 1u << k;
    }
  }
}

__device__ __forceinline__ void wait_flag(const int* f, int epoch) {
  while (ld_acquire(f) != epoch) __nanosleep(32);
}

// ============================================================================ a2: gradients
// SmartGD: the instances are in leaf nodes at the end of a tree, so the prediction is
// updated with the leaf weight of the node each instance ended in -- no tree traversal.
__global__ void k_grad(int64_t n, int loss, int first, double eta, double base,
                       const float* __restrict__ y, const double* __restrict__ wprev,
                       double* __restrict__ yhat, int32_t* __restrict__ pos,
                       double2* __restrict__ gh, double* __restrict__ partial) {
  double sg = 0.0, sh = 0.0;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += stride) {
    double yh = first ? base : __dadd_rn(yhat[i], __dmul_rn(eta, wprev[pos[i]]));
    yhat[i] = yh;
    const double yi = (double)y[i];
    double g, h;
    if (loss == GBDT_LOSS_SQUARED) {  // l = (y - yhat)^2: g = 2(yhat - y), h = 2 (R6)
      g = __dmul_rn(2.0, __dsub_rn(yh, yi));
      h = 2.0;
    } else {  // cross-entropy, reading R5
      const double p = __ddiv_rn(1.0, __dadd_rn(1.0, exp(-yh)));
      g = __dsub_rn(p, yi);
      const double hh = __dmul_rn(p, __dsub_rn(1.0, p));
      h = hh > 1e-16 ? hh : 1e-16;
    }
    gh[i] = make_double2(g, h);
    pos[i] = 0;
    sg += g;
    sh += h;
  }
  // fixed-shape block reduction (deterministic for a fixed grid)
  for (int o = 16; o; o >>= 1) {
    sg += __shfl_xor_sync(0xffffffffu, sg, o);
    sh += __shfl_xor_sync(0xffffffffu, sh, o);
  }
  __shared__ double wg[32], wh[32];
  if ((threadIdx.x & 31) == 0) { wg[threadIdx.x >> 5] = sg; wh[threadIdx.x >> 5] = sh; }
  __syncthreads();
  if (threadIdx.x == 0) {
    double a = 0.0, b = 0.0;
    for (int w = 0; w < (int)(blockDim.x >> 5); ++w) { a += wg[w]; b += wh[w]; }
    partial[2 * blockIdx.x] = a;
    partial[2 * blockIdx.x + 1] = b;
  }
}

// Root node totals + per-tree reset (single thread block).
__global__ void k_tree_begin(int nblk, const double* __restrict__ partial, int64_t n, double lam,
                             NodeTab root, int64_t NH, double* __restrict__ wcur,
                             uint8_t* __restrict__ hstate, gbdt_node* __restrict__ tree) {
  for (int64_t k = threadIdx.x; k < NH; k += blockDim.x) {
    wcur[k] = 0.0;
    hstate[k] = 0;
    gbdt_node z;
    z.heap_id = -1; z.is_leaf = 0; z.attr = -1; z.default_left = 0; z.split_value = 0.f;
    z.reserved = 0; z.gain = 0.0; z.G = 0.0; z.H = 0.0; z.weight = 0.0; z.count = 0;
    tree[k] = z;
  }
  if (threadIdx.x == 0) {
    double G = 0.0, H = 0.0;
    for (int b = 0; b < nblk; ++b) { G += partial[2 * b]; H += partial[2 * b + 1]; }
    *root.K = 1;
    root.heap[0] = 0;
    root.G[0] = G;
    root.H[0] = H;
    root.cnt[0] = (int32_t)n;
    root.pterm[0] = parent_term(G, H, lam);
  }
}

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

// ============================================================================ a3-a6: split find
template <bool kMissing, bool kTotals>
__global__ void __launch_bounds__(kThreads, 2) k_split_find(SplitArgs A) {
  __shared__ TileMeta sm;
  __shared__ SVf s_wtot[kWarps];
  __shared__ SVf s_wcar[kWarps];
  __shared__ AM s_mtot[kWarps];
  __shared__ AM s_mcar[kWarps];
  __shared__ unsigned char s_win[kTile];

  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int K = *A.t.Kp;
  const int epoch = *A.epochp;
  const int T = *A.t.tb.T;
  for (int i = tid; i < kTile; i += kThreads) s_win[i] = 0;

  for (;;) {
    if (tid == 0) {
      const int t = atomicAdd(A.t.counter, 1);
      sm.t = t;
      if (t < T) tile_meta(A.t, K, t, sm);
    }
    __syncthreads();
    const int t = sm.t;
    if (t >= T) break;
    const long long p0 = sm.p0, p1 = sm.p1;
    const long long base = p0 + (long long)tid * kItems;

    // ---------------------------------------------------------------- load (128-bit, blocked)
    float v[kItems];
    int id[kItems];
    float vnext = 0.f;
    unsigned vm = 0;
    if (base < p1) {
      const int4 i0 = __ldg(reinterpret_cast<const int4*>(A.t.ins + base));
      const int4 i1 = __ldg(reinterpret_cast<const int4*>(A.t.ins + base + 4));
      id[0] = i0.x; id[1] = i0.y; id[2] = i0.z; id[3] = i0.w;
      id[4] = i1.x; id[5] = i1.y; id[6] = i1.z; id[7] = i1.w;
      if (!kTotals) {
        const float4 v0 = __ldg(reinterpret_cast<const float4*>(A.t.val + base));
        const float4 v1 = __ldg(reinterpret_cast<const float4*>(A.t.val + base + 4));
        v[0] = v0.x; v[1] = v0.y; v[2] = v0.z; v[3] = v0.w;
        v[4] = v1.x; v[5] = v1.y; v[6] = v1.z; v[7] = v1.w;
        if (base + kItems < sm.colend) vnext = __ldg(A.t.val + base + kItems);
      } else {
#pragma unroll
        for (int k = 0; k < kItems; ++k) v[k] = 0.f;
      }
#pragma unroll
      for (int k = 0; k < kItems; ++k)
        if (base + k < p1) vm |= 1u << k;
    } else {
#pragma unroll
      for (int k = 0; k < kItems; ++k) { v[k] = 0.f; id[k] = 0; }
    }
    double g[kItems], h[kItems];
    int c[kItems];
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if ((vm >> k) & 1) {
        const double2 x = __ldg(A.gh + id[k]);  // random 16 B gather of (g_i, h_i)
        g[k] = x.x; h[k] = x.y;
      } else {
        g[k] = 0.0; h[k] = 0.0;
      }
    }
    int sj[kItems];
    unsigned hm, pem, rem;
    assign_segments<!kTotals>(A.t, sm, base, vm, v, vnext, sj, hm, pem, rem);

    // ---------------------------------------------------------------- segmented scan
    SVf run = svf_zero();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if ((vm >> k) & 1) {
        if ((hm >> k) & 1) { run.g = g[k]; run.h = h[k]; run.c = 1; run.f = 1; }
        else { run.g = run.g + g[k]; run.h = run.h + h[k]; run.c += 1; }
      }
      g[k] = run.g; h[k] = run.h; c[k] = run.c;
    }
    SVf inc = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const SVf y = shfl_up(inc, o);
      if (lane >= o) inc = comb(y, inc);
    }
    SVf exc = shfl_up(inc, 1);
    if (lane == 0) exc = svf_zero();
    if (lane == 31) s_wtot[wid] = inc;
    __syncthreads();
    if (wid == 0) {
      // in-tile fold of warp totals (fixed order), then the Fenwick look-back
      SVf agg = svf_zero();
      if (lane == 0) {
        for (int w = 0; w < kWarps; ++w) { s_wcar[w] = agg; agg = comb(agg, s_wtot[w]); }
      }
      agg = shfl_idx(agg, 0);
      const int u = sm.u;
      const int tb = t - u;
      const int jpub = __ffs(u + 1) - 1;  // top block of tile u covers (u - 2^jpub, u]
      // (1) publish this tile's Fenwick block first: it depends only on other tiles' blocks,
      //     never on any exclusive prefix, so the dependency depth stays <= log2(tiles)
      SVf got = svf_zero();
      if (lane < jpub) {
        const int tt = tb + u - (1 << lane);
        wait_flag(A.fw.E + tt, epoch);
        got = SVf{__ldcg(A.fw.G + tt), __ldcg(A.fw.H + tt), __ldcg(A.fw.C + tt), __ldcg(A.fw.F + tt)};
      }
      SVf B = agg;
      for (int i = 0; i < jpub; ++i) B = comb(shfl_idx(got, i), B);
      if (lane == 0) {
        A.fw.G[t] = B.g; A.fw.H[t] = B.h; A.fw.C[t] = B.c; A.fw.F[t] = B.f;
        st_release(A.fw.E + t, epoch);
      }
      // (2) exclusive prefix of the tile = fold of the Fenwick blocks covering [0, u)
      const int pc = __popc(u);
      SVf q = svf_zero();
      if (lane < pc) {
        int i = u;
        for (int r = 0; r < lane; ++r) i &= i - 1;
        const int tt = tb + i - 1;
        wait_flag(A.fw.E + tt, epoch);
        q = SVf{__ldcg(A.fw.G + tt), __ldcg(A.fw.H + tt), __ldcg(A.fw.C + tt), __ldcg(A.fw.F + tt)};
      }
      SVf E = svf_zero();
      for (int b = pc - 1; b >= 0; --b) E = comb(E, shfl_idx(q, b));
      __syncwarp();
      if (lane < kWarps) s_wcar[lane] = comb(E, s_wcar[lane]);
    }
    __syncthreads();
    {
      const SVf car = comb(s_wcar[wid], exc);
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        const bool head_before = (hm & ((2u << k) - 1u)) != 0u;
        if (!head_before) { g[k] = car.g + g[k]; h[k] = car.h + h[k]; c[k] = car.c + c[k]; }
      }
    }

    if (kTotals) {
      // present totals of each segment = inclusive prefix at its last entry
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (((vm & rem) >> k) & 1) {
          const long long s = sm.sb + sj[k];
          A.segPG_out[s] = g[k];
          A.segPH_out[s] = h[k];
        }
      }
      __syncthreads();
      continue;
    }

    // ---------------------------------------------------------------- gains at run ends
    double gn[kItems];
    unsigned dm = 0, okm = 0;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      gn[k] = 0.0;
      if (!(((vm & rem) >> k) & 1)) continue;
      const int j = sj[k];
      const double Gt = A.nodes.G[j], Ht = A.nodes.H[j], pt = A.nodes.pterm[j];
      const int Ct = A.nodes.cnt[j];
      const int cL = c[k];
      bool ok = false;
      double best = 0.0;
      int bd = 0;
      if (cL >= 1 && Ct - cL >= 1) { best = eq2_gain(g[k], h[k], Gt, Ht, A.lam, pt); ok = true; }
      if (kMissing) {
        const long long s = sm.sb + j;
        const int cM = Ct - (int)A.t.tb.seg_cnt[s];
        if (cM > 0) {
          const double GM = Gt - A.segPG[s], HM = Ht - A.segPH[s];
          const int cL1 = cL + cM;
          if (cL1 >= 1 && Ct - cL1 >= 1) {
            const double g1 = eq2_gain(g[k] + GM, h[k] + HM, Gt, Ht, A.lam, pt);
            if (!ok || g1 > best) { best = g1; bd = 1; ok = true; }
          }
        }
      }
      gn[k] = best;
      dm |= (unsigned)bd << k;
      okm |= (unsigned)ok << k;
    }

    // ---------------------------------------------------------------- per-piece argmax scan
    const int ibase = tid * kItems;
    AM mrun = am_none();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1)) continue;
      AM it;
      it.gain = gn[k]; it.value = v[k];
      it.meta = (ibase + k) | (int)(((dm >> k) & 1) << 12) | (int)(((okm >> k) & 1) << 13);
      it.f = ((hm >> k) & 1) || (tid == 0 && k == 0);
      mrun = am_comb(mrun, it);
    }
    AM minc = mrun;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const AM y = shfl_up(minc, o);
      if (lane >= o) minc = am_comb(y, minc);
    }
    AM mexc = shfl_up(minc, 1);
    if (lane == 0) mexc = am_none();
    if (lane == 31) s_mtot[wid] = minc;
    __syncthreads();
    if (tid == 0) {
      AM acc = am_none();
      for (int w = 0; w < kWarps; ++w) { s_mcar[w] = acc; acc = am_comb(acc, s_mtot[w]); }
    }
    __syncthreads();
    {
      AM r = am_comb(s_mcar[wid], mexc);
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (!((vm >> k) & 1)) continue;
        AM it;
        it.gain = gn[k]; it.value = v[k];
        it.meta = (ibase + k) | (int)(((dm >> k) & 1) << 12) | (int)(((okm >> k) & 1) << 13);
        it.f = ((hm >> k) & 1) || (tid == 0 && k == 0);
        r = am_comb(r, it);
        if (((pem >> k) & 1) && am_valid(r)) s_win[r.meta & 0xfff] = 1;
      }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1) || !s_win[ibase + k]) continue;
      s_win[ibase + k] = 0;
      const int j = sj[k];
      const long long s = sm.sb + j;
      Rec r;
      r.gain = gn[k];
      r.value = v[k];
      r.attr = A.t.a_base + sm.a;
      r.dir = (dm >> k) & 1;
      r.node = j;
      r.epoch = epoch;
      r.shard = A.shard;
      r.pos = base + k;
      if (r.dir) {
        const int Ct = A.nodes.cnt[j];
        const int cM = Ct - (int)A.t.tb.seg_cnt[s];
        r.GL = g[k] + (A.nodes.G[j] - A.segPG[s]);
        r.HL = h[k] + (A.nodes.H[j] - A.segPH[s]);
        r.cntL = c[k] + cM;
      } else {
        r.GL = g[k]; r.HL = h[k]; r.cntL = c[k];
      }
      const int slot = atomicAdd(A.nrec, 1);
      A.rec[slot] = r;
      atomicMax(A.gkey + j, gain_key(r.gain));
    }
    __syncthreads();
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
  double* hweight;      // by heap id (this tree)
  gbdt_node* tree;
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
                       const int32_t* __restrict__ ins, uint8_t* __restrict__ bits) {
  const int K = *Kp;
  const int j = blockIdx.y;
  if (j >= K || cidx[j] < 0) return;
  const Rec& w = winner[j];
  if (w.shard != shard) return;
  const long long s = (long long)(w.attr - a_base) * K + j;
  const long long s0 = tb.seg_start[s], n = tb.seg_cnt[s];
  const int defhi = w.dir;
  for (long long q = (long long)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (long long)gridDim.x * blockDim.x) {
    const long long p = s0 + q;
    const int high = p <= w.pos;   // prefix of the descending list = values >= split value
    if (high != defhi) bits[ins[p]] = 1;  // goes to the non-default side
  }
}

__global__ void k_nodemap(int64_t n, const uint8_t* __restrict__ bits, const uint8_t* __restrict__ hstate,
                          const uint8_t* __restrict__ hdef, int32_t* __restrict__ pos,
                          uint8_t* __restrict__ side) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int h = pos[i];
    uint8_t sd = 0;
    if (hstate[h] == 1) {
      const int defhi = hdef[h];
      const int hi = bits[i] ? !defhi : defhi;
      pos[i] = hi ? 2 * h + 1 : 2 * h + 2;
      sd = hi ? 1 : 2;
    }
    side[i] = sd;
  }
}

// ============================================================================ a8: partition
__global__ void __launch_bounds__(kThreads) k_part_count(PartArgs A) {
  constexpr int kSlots = 512;
  __shared__ TileMeta sm;
  __shared__ unsigned s_cnt[kSlots];
  __shared__ unsigned s_red[kWarps];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int K = *A.t.Kp;
  const int T = *A.t.tb.T;
  for (;;) {
    if (tid == 0) {
      const int t = atomicAdd(A.t.counter, 1);
      sm.t = t;
      if (t < T) tile_meta(A.t, K, t, sm);
    }
    __syncthreads();
    const int t = sm.t;
    if (t >= T) break;
    const int nslots = sm.jlast - sm.j0 + 1;
    for (int i = tid; i < min(nslots, kSlots); i += kThreads) s_cnt[i] = 0;
    __syncthreads();
    const long long base = sm.p0 + (long long)tid * kItems;
    unsigned vm = 0;
    int id[kItems];
    if (base < sm.p1) {
      const int4 i0 = __ldg(reinterpret_cast<const int4*>(A.t.ins + base));
      const int4 i1 = __ldg(reinterpret_cast<const int4*>(A.t.ins + base + 4));
      id[0] = i0.x; id[1] = i0.y; id[2] = i0.z; id[3] = i0.w;
      id[4] = i1.x; id[5] = i1.y; id[6] = i1.z; id[7] = i1.w;
#pragma unroll
      for (int k = 0; k < kItems; ++k)
        if (base + k < sm.p1) vm |= 1u << k;
    }
    float dummy[kItems];
    int sj[kItems];
    unsigned hm, pem, rem;
    assign_segments<false>(A.t, sm, base, vm, dummy, 0.f, sj, hm, pem, rem);
    unsigned tot = 0;
    // thread-local run-length accumulation per segment, flushed to shared slots
    unsigned acc = 0;
    int cur = -1;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1)) continue;
      const uint8_t sd = A.side[id[k]];
      const unsigned x = sd == 1 ? 1u : (sd == 2 ? (1u << 16) : 0u);
      tot += x;
      if (sj[k] != cur) {
        if (cur >= 0 && acc) {
          const int slot = cur - sm.j0;
          if (slot < kSlots) atomicAdd(&s_cnt[slot], acc);
          else { atomicAdd(A.segH + sm.sb + cur, (int)(acc & 0xffffu)); atomicAdd(A.segL + sm.sb + cur, (int)(acc >> 16)); }
        }
        cur = sj[k];
        acc = 0;
      }
      acc += x;
    }
    if (cur >= 0 && acc) {
      const int slot = cur - sm.j0;
      if (slot < kSlots) atomicAdd(&s_cnt[slot], acc);
      else { atomicAdd(A.segH + sm.sb + cur, (int)(acc & 0xffffu)); atomicAdd(A.segL + sm.sb + cur, (int)(acc >> 16)); }
    }
    for (int o = 16; o; o >>= 1) tot += __shfl_xor_sync(0xffffffffu, tot, o);
    if (lane == 0) s_red[wid] = tot;
    __syncthreads();
    if (tid == 0) {
      unsigned s = 0;
      for (int w = 0; w < kWarps; ++w) s += s_red[w];
      A.tile_cnt[t] = s;
    }
    for (int i = tid; i < min(nslots, kSlots); i += kThreads) {
      const unsigned x = s_cnt[i];
      if (x) {
        atomicAdd(A.segH + sm.sb + sm.j0 + i, (int)(x & 0xffffu));
        atomicAdd(A.segL + sm.sb + sm.j0 + i, (int)(x >> 16));
      }
    }
    __syncthreads();
  }
}

struct PlanArgs {
  int m;
  const int32_t* Kp;      // current K
  const int32_t* Knp;     // next K
  const int32_t* cidx;
  const int32_t* Tp;      // current tiles
  const uint32_t* tile_cnt;
  const int32_t* segH;
  const int32_t* segL;
  unsigned long long* tile_pre;
  unsigned long long* seg_pre;
  int64_t* out_hi;
  int64_t* out_lo;
  int64_t* len_tmp;       // [m]
  Tables nxt;
};

// Single thread block: prefix sums that place every child segment (stable, attribute-major,
// children in heap order) and the next level's tile table.
__global__ void __launch_bounds__(1024) k_part_plan(PlanArgs A) {
  const int K = *A.Kp, Kn = *A.Knp, T = *A.Tp, m = A.m;
  unsigned long long carry = 0, tot;
  for (int base = 0; base < T; base += blockDim.x) {
    const int i = base + threadIdx.x;
    unsigned long long x = 0;
    if (i < T) { const unsigned c = A.tile_cnt[i]; x = (unsigned long long)(c & 0xffffu) | ((unsigned long long)(c >> 16) << 32); }
    const unsigned long long ex = block_exscan_u64(x, tot);
    if (i < T) A.tile_pre[i] = carry + ex;
    carry += tot;
  }
  const long long S = (long long)m * K;
  carry = 0;
  for (long long base = 0; base < S; base += blockDim.x) {
    const long long s = base + threadIdx.x;
    unsigned long long x = 0;
    if (s < S) x = (unsigned long long)(unsigned)A.segH[s] | ((unsigned long long)(unsigned)A.segL[s] << 32);
    const unsigned long long ex = block_exscan_u64(x, tot);
    if (s < S) A.seg_pre[s] = carry + ex;
    carry += tot;
  }
  for (int a = threadIdx.x; a < m; a += blockDim.x) {
    long long L = 0;
    for (int j = 0; j < K; ++j)
      if (A.cidx[j] >= 0) L += (long long)A.segH[(long long)a * K + j] + A.segL[(long long)a * K + j];
    A.len_tmp[a] = L;
    A.nxt.col_len[a] = L;
  }
  __syncthreads();
  unsigned long long cpos = 0, ctile = 0, t1, t2;
  for (int base = 0; base < m; base += blockDim.x) {
    const int a = base + threadIdx.x;
    unsigned long long L = a < m ? (unsigned long long)A.len_tmp[a] : 0ull;
    const unsigned long long xp = (L + 3) & ~3ull;
    const unsigned long long xt = (L + kTile - 1) / kTile;
    const unsigned long long ep = block_exscan_u64(xp, t1);
    const unsigned long long et = block_exscan_u64(xt, t2);
    if (a < m) { A.nxt.col_start[a] = (int64_t)(cpos + ep); A.nxt.tile_start[a] = (int32_t)(ctile + et); }
    cpos += t1;
    ctile += t2;
  }
  if (threadIdx.x == 0) {
    A.nxt.col_start[m] = (int64_t)cpos;
    A.nxt.tile_start[m] = (int32_t)ctile;
    *A.nxt.T = (int32_t)ctile;
  }
  __syncthreads();
  for (int a = threadIdx.x; a < m; a += blockDim.x) {
    long long r = A.nxt.col_start[a];
    for (int j = 0; j < K; ++j) {
      const int c = A.cidx[j];
      if (c < 0) continue;
      const long long s = (long long)a * K + j;
      const long long hi = A.segH[s], lo = A.segL[s];
      A.out_hi[s] = r;
      A.nxt.seg_start[(long long)a * Kn + c] = r;
      A.nxt.seg_cnt[(long long)a * Kn + c] = hi;
      r += hi;
      A.out_lo[s] = r;
      A.nxt.seg_start[(long long)a * Kn + c + 1] = r;
      A.nxt.seg_cnt[(long long)a * Kn + c + 1] = lo;
      r += lo;
    }
  }
}

__global__ void __launch_bounds__(kThreads) k_part_scatter(PartArgs A) {
  __shared__ TileMeta sm;
  __shared__ unsigned s_w[kWarps];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int K = *A.t.Kp;
  const int T = *A.t.tb.T;
  for (;;) {
    if (tid == 0) {
      const int t = atomicAdd(A.t.counter, 1);
      sm.t = t;
      if (t < T) tile_meta(A.t, K, t, sm);
    }
    __syncthreads();
    const int t = sm.t;
    if (t >= T) break;
    const long long base = sm.p0 + (long long)tid * kItems;
    unsigned vm = 0;
    int id[kItems];
    float v[kItems];
    if (base < sm.p1) {
      const int4 i0 = __ldg(reinterpret_cast<const int4*>(A.t.ins + base));
      const int4 i1 = __ldg(reinterpret_cast<const int4*>(A.t.ins + base + 4));
      const float4 v0 = __ldg(reinterpret_cast<const float4*>(A.t.val + base));
      const float4 v1 = __ldg(reinterpret_cast<const float4*>(A.t.val + base + 4));
      id[0] = i0.x; id[1] = i0.y; id[2] = i0.z; id[3] = i0.w;
      id[4] = i1.x; id[5] = i1.y; id[6] = i1.z; id[7] = i1.w;
      v[0] = v0.x; v[1] = v0.y; v[2] = v0.z; v[3] = v0.w;
      v[4] = v1.x; v[5] = v1.y; v[6] = v1.z; v[7] = v1.w;
#pragma unroll
      for (int k = 0; k < kItems; ++k)
        if (base + k < sm.p1) vm |= 1u << k;
    }
    int sj[kItems];
    unsigned hm, pem, rem;
    assign_segments<false>(A.t, sm, base, vm, v, 0.f, sj, hm, pem, rem);
    uint8_t sd[kItems];
    unsigned loc = 0;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      sd[k] = ((vm >> k) & 1) ? A.side[id[k]] : 0;
      loc += sd[k] == 1 ? 1u : (sd[k] == 2 ? (1u << 16) : 0u);
    }
    unsigned inc = loc;
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned y = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += y;
    }
    if (lane == 31) s_w[wid] = inc;
    __syncthreads();
    unsigned wex = 0;
    for (int w = 0; w < wid; ++w) wex += s_w[w];
    unsigned ex = wex + inc - loc;  // exclusive packed count before this thread's first item
    const unsigned long long tp = A.tile_pre[t];
    const long long chi0 = (long long)(tp & 0xffffffffull), clo0 = (long long)(tp >> 32);
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (sd[k]) {
        const long long s = sm.sb + sj[k];
        const unsigned long long sp = A.seg_pre[s];
        long long dst;
        if (sd[k] == 1) dst = A.out_hi[s] + (chi0 + (long long)(ex & 0xffffu) - (long long)(sp & 0xffffffffull));
        else dst = A.out_lo[s] + (clo0 + (long long)(ex >> 16) - (long long)(sp >> 32));
        A.val_out[dst] = v[k];
        A.ins_out[dst] = id[k];
        ex += sd[k] == 1 ? 1u : (1u << 16);
      }
    }
    __syncthreads();
  }
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

struct ShardWork {
  DBuf mem;
  Tables tab[2];
  Fenwick fw;
  int32_t* fwE2;  // publication flags of the segment-totals pass
  Rec* rec;
  int* nrec;
  unsigned long long *gkey, *tkey;
  uint32_t* tile_cnt;
  unsigned long long* tile_pre;
  int32_t *segH, *segL;
  unsigned long long* seg_pre;
  int64_t *out_hi, *out_lo, *len_tmp;
  double *segPG, *segPH;
  int* counters;  // [4]
};

struct PhaseTimer {
  bool on = false;
  cudaStream_t st = nullptr;
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> ev;
  int cur = -1;
  cudaEvent_t e0 = nullptr;
  void begin(int phase) {
    if (!on) return;
    cudaEvent_t a;
    GBDT_CUDA(cudaEventCreate(&a));
    GBDT_CUDA(cudaEventRecord(a, st));
    cur = phase;
    e0 = a;
  }
  void end() {
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

void train(Dataset& ds, const gbdt_params& P, Model& model, double* margin_out) {
  GBDT_CUDA(cudaSetDevice(ds.device));
  cudaStream_t st = ds.stream;
  launches_reset();
  const int d = P.max_depth;
  const int64_t NH = (int64_t(1) << (d + 1)) - 1;
  const int Kcap = 1 << (d - 1);
  const int64_t n = ds.n;
  const int nloc = (int)ds.shards.size();
  const int nsh = ds.n_total_shards;
  int sms = 148;
  GBDT_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, ds.device));
  int occ = 1;
  GBDT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_split_find<false, false>, kThreads, 0));
  const unsigned tile_grid = (unsigned)(sms * std::max(occ, 1));
  int occp = 1;
  GBDT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occp, k_part_scatter, kThreads, 0));
  const unsigned part_grid = (unsigned)(sms * std::max(occp, 1));
  const unsigned inst_grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), (int64_t)sms * 8));
  const int grad_blocks = (int)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), (int64_t)sms * 4));

  // ---------------------------------------------------------------- per-device state
  Carve cv{nullptr};
  auto sz_dev = [&](Carve& c) {
    c.take<double2>(n); c.take<double>(n); c.take<int32_t>(n); c.take<uint8_t>(n); c.take<uint8_t>(n);
    c.take<double>(2 * NH); c.take<uint8_t>(NH); c.take<uint8_t>(NH);
    c.take<gbdt_node>((size_t)P.n_trees * NH); c.take<double>(2 * grad_blocks);
    for (int b = 0; b < 2; ++b) { c.take<int32_t>(1); c.take<int32_t>(Kcap); c.take<double>(Kcap); c.take<double>(Kcap); c.take<int32_t>(Kcap); c.take<double>(Kcap); }
    c.take<int32_t>(Kcap); c.take<Rec>(Kcap); c.take<Rec>((size_t)nsh * Kcap); c.take<int>(1);
    c.take<unsigned long long>((size_t)nloc * Kcap); c.take<unsigned long long>((size_t)nloc * Kcap);
    c.take<int>(nloc);
  };
  Carve probe{nullptr};
  sz_dev(probe);
  DBuf dmem(probe.off + 1024, st);
  GBDT_CUDA(cudaMemsetAsync(dmem.p, 0, dmem.bytes, st));
  Carve c{dmem.as<char>()};
  double2* gh = c.take<double2>(n);
  double* yhat = c.take<double>(n);
  int32_t* pos = c.take<int32_t>(n);
  uint8_t* side = c.take<uint8_t>(n);
  uint8_t* bits = c.take<uint8_t>(n);
  double* hweight = c.take<double>(2 * NH);
  uint8_t* hstate = c.take<uint8_t>(NH);
  uint8_t* hdef = c.take<uint8_t>(NH);
  gbdt_node* trees = c.take<gbdt_node>((size_t)P.n_trees * NH);
  double* partial = c.take<double>(2 * grad_blocks);
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

  // ---------------------------------------------------------------- per-shard state
  std::vector<ShardWork> sw(nloc);
  for (int li = 0; li < nloc; ++li) {
    Shard& sh = *ds.shards[li];
    ShardWork& w = sw[li];
    const int m = sh.m;
    const int64_t S = (int64_t)m * Kcap;
    const int64_t T0 = std::max(sh.T0, 1);
    auto sz = [&](Carve& q) {
      for (int b = 0; b < 2; ++b) {
        q.take<int64_t>(m + 1); q.take<int64_t>(m); q.take<int32_t>(m + 1); q.take<int64_t>(S); q.take<int64_t>(S); q.take<int32_t>(1);
      }
      q.take<double>(T0); q.take<double>(T0); q.take<int32_t>(T0); q.take<int32_t>(T0); q.take<int32_t>(T0);
      q.take<int32_t>(T0);
      q.take<Rec>(T0 + S); q.take<uint32_t>(T0); q.take<unsigned long long>(T0);
      q.take<int32_t>(S); q.take<int32_t>(S); q.take<unsigned long long>(S); q.take<int64_t>(S); q.take<int64_t>(S);
      q.take<int64_t>(m); q.take<double>(S); q.take<double>(S); q.take<int>(4);
    };
    Carve pq{nullptr};
    sz(pq);
    w.mem.alloc(pq.off + 1024, st);
    GBDT_CUDA(cudaMemsetAsync(w.mem.p, 0, w.mem.bytes, st));
    Carve q{w.mem.as<char>()};
    for (int b = 0; b < 2; ++b) {
      w.tab[b].col_start = q.take<int64_t>(m + 1); w.tab[b].col_len = q.take<int64_t>(m);
      w.tab[b].tile_start = q.take<int32_t>(m + 1); w.tab[b].seg_start = q.take<int64_t>(S);
      w.tab[b].seg_cnt = q.take<int64_t>(S); w.tab[b].T = q.take<int32_t>(1);
    }
    w.fw.G = q.take<double>(T0); w.fw.H = q.take<double>(T0); w.fw.C = q.take<int32_t>(T0);
    w.fw.F = q.take<int32_t>(T0); w.fw.E = q.take<int32_t>(T0);
    w.fwE2 = q.take<int32_t>(T0);
    w.rec = q.take<Rec>(T0 + S);
    w.tile_cnt = q.take<uint32_t>(T0);
    w.tile_pre = q.take<unsigned long long>(T0);
    w.segH = q.take<int32_t>(S); w.segL = q.take<int32_t>(S);
    w.seg_pre = q.take<unsigned long long>(S);
    w.out_hi = q.take<int64_t>(S); w.out_lo = q.take<int64_t>(S);
    w.len_tmp = q.take<int64_t>(m);
    w.segPG = q.take<double>(S); w.segPH = q.take<double>(S);
    w.counters = q.take<int>(4);
    w.nrec = nrec + li;
    w.gkey = gkey + (size_t)li * Kcap;
    w.tkey = tkey + (size_t)li * Kcap;
  }

  PhaseTimer tm;
  tm.on = P.profile != 0;
  tm.st = st;
  cudaEvent_t tot0 = nullptr, tot1 = nullptr;
  if (tm.on) {
    GBDT_CUDA(cudaEventCreate(&tot0));
    GBDT_CUDA(cudaEventCreate(&tot1));
    GBDT_CUDA(cudaEventRecord(tot0, st));
  }
  const double thr = P.gamma > 0 ? P.gamma : 0.0;

  for (int t = 0; t < P.n_trees; ++t) {
    double* wprev = hweight + (size_t)((t + 1) & 1) * NH;
    double* wcur = hweight + (size_t)(t & 1) * NH;
    gbdt_node* tree = trees + (size_t)t * NH;
    tm.begin(GBDT_PHASE_GRAD);
    k_grad<<<grad_blocks, 256, 0, st>>>(n, P.loss, t == 0, P.eta, P.base_margin, ds.y.as<float>(), wprev,
                                        yhat, pos, gh, partial);
    GBDT_LAUNCH_CHECK();
    k_tree_begin<<<1, 1024, 0, st>>>(grad_blocks, partial, n, P.lambda, nt[0], NH, wcur, hstate, tree);
    GBDT_LAUNCH_CHECK();
    count_launch(2);
    tm.end();

    for (int lvl = 0; lvl < d; ++lvl) {
      NodeTab& cur = nt[lvl & 1];
      NodeTab& nxt = nt[(lvl + 1) & 1];
      const bool last = (lvl == d - 1);
      const int Kl = 1 << lvl;  // upper bound of active nodes at this level
      tm.begin(GBDT_PHASE_DECIDE);
      k_level_begin<<<1, 1024, 0, st>>>(epoch, sw[0].counters, 0, nrec, nloc, cur.K, gkey, tkey, Kcap);
      GBDT_LAUNCH_CHECK();
      count_launch();
      for (int li = 0; li < nloc; ++li) GBDT_CUDA(cudaMemsetAsync(sw[li].counters, 0, 4 * sizeof(int), st));
      tm.end();
      tm.begin(GBDT_PHASE_SPLIT_FIND);
      for (int li = 0; li < nloc; ++li) {
        Shard& sh = *ds.shards[li];
        ShardWork& w = sw[li];
        if (sh.m == 0) continue;
        const Tables tb = lvl == 0 ? sh.root : w.tab[lvl & 1];
        const float* val = lvl == 0 ? sh.val0.as<float>() : sh.valw[lvl & 1].as<float>();
        const int32_t* ins = lvl == 0 ? sh.ins0.as<int32_t>() : sh.insw[lvl & 1].as<int32_t>();
        SplitArgs A;
        A.t = TileArgs{val, ins, tb, sh.m, sh.a_begin, cur.K, w.counters};
        A.gh = gh; A.nodes = cur; A.segPG = w.segPG; A.segPH = w.segPH; A.lam = P.lambda;
        A.epochp = epoch; A.fw = w.fw; A.rec = w.rec; A.nrec = w.nrec; A.gkey = w.gkey; A.shard = sh.index;
        A.totals_only = 0; A.segPG_out = w.segPG; A.segPH_out = w.segPH;
        if (ds.has_missing) {
          // present totals per segment first (needed for the missing direction); own
          // tile counter and own Fenwick publication flags, same level epoch
          SplitArgs AT = A;
          AT.t.counter = w.counters + 3;
          AT.fw.E = w.fwE2;
          k_split_find<true, true><<<tile_grid, kThreads, 0, st>>>(AT);
          GBDT_LAUNCH_CHECK();
          count_launch();
          k_split_find<true, false><<<tile_grid, kThreads, 0, st>>>(A);
        } else {
          k_split_find<false, false><<<tile_grid, kThreads, 0, st>>>(A);
        }
        GBDT_LAUNCH_CHECK();
        count_launch();
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
      if (ds.comm && ds.comm->world > 1) {
        tm.begin(GBDT_PHASE_COMM);
        Rec* mine = best_all + (size_t)ds.shards[0]->index * Kcap;
        ds.comm->allgather(mine, best_all, sizeof(Rec) * Kcap, st);
        tm.end();
      }
      tm.begin(GBDT_PHASE_DECIDE);
      DecideArgs D;
      D.cur = cur; D.nxt = nxt; D.best_all = best_all; D.nshard = nsh; D.Kcap = Kcap; D.epochp = epoch;
      D.lam = P.lambda; D.thr = thr; D.last_level = last; D.cidx = cidx; D.winner = winner;
      D.hstate = hstate; D.hdef = hdef; D.hweight = wcur; D.tree = tree;
      k_decide<<<1, 1024, 0, st>>>(D);
      GBDT_LAUNCH_CHECK();
      count_launch();
      tm.end();

      tm.begin(GBDT_PHASE_NODEMAP);
      GBDT_CUDA(cudaMemsetAsync(bits, 0, (size_t)n, st));
      for (int li = 0; li < nloc; ++li) {
        Shard& sh = *ds.shards[li];
        if (sh.m == 0) continue;
        const Tables tb = lvl == 0 ? sh.root : sw[li].tab[lvl & 1];
        const int32_t* ins = lvl == 0 ? sh.ins0.as<int32_t>() : sh.insw[lvl & 1].as<int32_t>();
        dim3 grid((unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256 * (int64_t)Kl), (int64_t)sms * 4)), (unsigned)Kl);
        k_mark<<<grid, 256, 0, st>>>(cur.K, cidx, winner, sh.index, sh.a_begin, tb, ins, bits);
        GBDT_LAUNCH_CHECK();
        count_launch();
      }
      tm.end();
      if (ds.comm && ds.comm->world > 1) {
        tm.begin(GBDT_PHASE_COMM);
        ds.comm->allreduce_sum_u8(bits, (size_t)n, st);
        tm.end();
      }
      tm.begin(GBDT_PHASE_NODEMAP);
      k_nodemap<<<inst_grid, 256, 0, st>>>(n, bits, hstate, hdef, pos, side);
      GBDT_LAUNCH_CHECK();
      count_launch();
      tm.end();

      if (last) break;
      tm.begin(GBDT_PHASE_PARTITION);
      for (int li = 0; li < nloc; ++li) {
        Shard& sh = *ds.shards[li];
        ShardWork& w = sw[li];
        if (sh.m == 0) continue;
        const Tables tb = lvl == 0 ? sh.root : w.tab[lvl & 1];
        const Tables tn = w.tab[(lvl + 1) & 1];
        const float* val = lvl == 0 ? sh.val0.as<float>() : sh.valw[lvl & 1].as<float>();
        const int32_t* ins = lvl == 0 ? sh.ins0.as<int32_t>() : sh.insw[lvl & 1].as<int32_t>();
        const size_t Sl = (size_t)sh.m * Kl;
        GBDT_CUDA(cudaMemsetAsync(w.segH, 0, Sl * 4, st));
        GBDT_CUDA(cudaMemsetAsync(w.segL, 0, Sl * 4, st));
        PartArgs PA;
        PA.t = TileArgs{val, ins, tb, sh.m, sh.a_begin, cur.K, w.counters + 1};
        PA.side = side; PA.tile_cnt = w.tile_cnt; PA.segH = w.segH; PA.segL = w.segL;
        PA.tile_pre = w.tile_pre; PA.seg_pre = w.seg_pre; PA.out_hi = w.out_hi; PA.out_lo = w.out_lo;
        PA.val_out = sh.valw[(lvl + 1) & 1].as<float>();
        PA.ins_out = sh.insw[(lvl + 1) & 1].as<int32_t>();
        k_part_count<<<part_grid, kThreads, 0, st>>>(PA);
        GBDT_LAUNCH_CHECK();
        PlanArgs PL;
        PL.m = sh.m; PL.Kp = cur.K; PL.Knp = nxt.K; PL.cidx = cidx; PL.Tp = tb.T; PL.tile_cnt = w.tile_cnt;
        PL.segH = w.segH; PL.segL = w.segL; PL.tile_pre = w.tile_pre; PL.seg_pre = w.seg_pre;
        PL.out_hi = w.out_hi; PL.out_lo = w.out_lo; PL.len_tmp = w.len_tmp; PL.nxt = tn;
        k_part_plan<<<1, 1024, 0, st>>>(PL);
        GBDT_LAUNCH_CHECK();
        PA.t.counter = w.counters + 2;
        k_part_scatter<<<part_grid, kThreads, 0, st>>>(PA);
        GBDT_LAUNCH_CHECK();
        count_launch(3);
      }
      tm.end();
    }
  }
  // final SmartGD step: the last tree's leaf weights
  {
    double* wlast = hweight + (size_t)((P.n_trees - 1) & 1) * NH;
    k_apply<<<inst_grid, 256, 0, st>>>(n, P.eta, wlast, pos, yhat);
    GBDT_LAUNCH_CHECK();
    count_launch();
  }
  if (tm.on) GBDT_CUDA(cudaEventRecord(tot1, st));
  model.n_trees = P.n_trees;
  model.max_depth = d;
  model.loss = P.loss;
  model.n_cols = ds.m;
  model.eta = P.eta;
  model.base_margin = P.base_margin;
  model.lambda = P.lambda;
  model.device = ds.device;
  model.nodes.resize((size_t)P.n_trees * NH);
  GBDT_CUDA(cudaMemcpyAsync(model.nodes.data(), trees, sizeof(gbdt_node) * model.nodes.size(),
                            cudaMemcpyDeviceToHost, st));
  if (margin_out)
    GBDT_CUDA(cudaMemcpyAsync(margin_out, yhat, sizeof(double) * (size_t)n, cudaMemcpyDeviceToHost, st));
  GBDT_CUDA(cudaStreamSynchronize(st));
  for (int i = 0; i < GBDT_N_PHASES; ++i) model.timings[i] = 0.0;
  if (tm.on) {
    tm.collect(model.timings);
    float tt = 0;
    GBDT_CUDA(cudaEventElapsedTime(&tt, tot0, tot1));
    model.timings[GBDT_PHASE_TOTAL] = tt;
    cudaEventDestroy(tot0);
    cudaEventDestroy(tot1);
  }
}

}  // namespace gbdt
