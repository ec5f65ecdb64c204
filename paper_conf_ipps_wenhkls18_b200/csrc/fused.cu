// fused.cu -- dense levels below the root: the partition of level l and the split
// finding of level l+1 in one streaming pass over the level's lists.
//
// For data without missing values every (node, attribute) segment of node j holds exactly the
// node's cnt[j] instances, so a child's segment is its side of the parent's segment, in the
// parent's order (order preserving), and the child's segmented prefix sums (P:197-208,
// Fig. 1) can be formed while the parent's entries stream past.  A level is cut into 2048-entry
// TILES (attribute-aligned; tile k of an attribute covers its list positions [2048 k, 2048 k +
// 2048) at that level, whatever the sharding) and runs in three steps:
//
//   k_tile_agg   per tile: every entry's child side -- the node's decision (leaf -> dropped) and,
//                for a split node, one bit gathered from the instance -> high-child bitmap
//                -- kept as a bit per entry, and the tile's per-side count, exact fixed-point
//                (g, h) sums and last entry of its LAST segment piece
//   k_tscan1/2/3 the exact segmented inclusive scan of those records over the tiles (integer sums:
//                any decomposition gives the same carries)
//   k_fused      per tile, TMA-staged in shared memory (2-stage ring): a stable in-tile partition by
//                (segment, side) ranked by a block scan of the packed side counts (the tile becomes
//                contiguous runs of CHILD entries in child order), the segmented prefix sums of
//                (g, h) over those runs from the carry of the tiles before, Eq. 2 (+lambda,
//                reading R1) at every boundary between two distinct values of a child segment (run
//                ends), the per-child-node argmax in the R12 total order, and the child
//                runs written to the next level's lists (coalesced) unless the children are the
//                last level that splits
//   k_mark_fused the instance -> child bits of a level found by k_fused: the winner's child
//                segment is the winner's side of its parent segment in the PARENT level's lists,
//                and the high part of it is every such entry at a parent position <= Rec.pos
//
// Determinism: inside a tile every sum has a fixed association, and carries are exact integer
// sums, so every gain -- hence every tree -- is bit-identical for any attribute sharding.
#include <algorithm>
#include <climits>

#include "kernels.cuh"

namespace gbdt {
namespace {

constexpr int kFT = 256;            // threads per CTA
constexpr int kFI = 8;              // items per thread (blocked arrangement)
constexpr int kFTile = kFT * kFI;   // entries per tile
constexpr int kFW = kFT / 32;
constexpr int kTSGroup = 256;       // tiles per CTA in the tile scan
constexpr int kFusedMaxCTAs = 148 * 8;  // persistent k_fused CTAs (node-best scratch per CTA)
#ifndef GBDT_FUSED_STAGES
#define GBDT_FUSED_STAGES 1
#endif
#ifndef GBDT_FUSED_CTAS
#define GBDT_FUSED_CTAS 3
#endif
constexpr int kFS = GBDT_FUSED_STAGES;

static_assert(sizeof(TRec) == 96, "tile record");

__device__ __forceinline__ unsigned __int128 u128(unsigned long long lo, unsigned long long hi) {
  return ((unsigned __int128)hi << 64) | lo;
}
// x (+) y: y follows x in list order
__device__ __forceinline__ TSide tside_add(const TSide& x, const TSide& y) {
  TSide r;
  const unsigned __int128 G = u128(x.g_lo, x.g_hi) + u128(y.g_lo, y.g_hi);
  const unsigned __int128 H = u128(x.h_lo, x.h_hi) + u128(y.h_lo, y.h_hi);
  r.g_lo = (unsigned long long)G; r.g_hi = (unsigned long long)(G >> 64);
  r.h_lo = (unsigned long long)H; r.h_hi = (unsigned long long)(H >> 64);
  r.cnt = x.cnt + y.cnt;
  r.val = y.cnt ? y.val : x.val;
  r.pos = y.cnt ? y.pos : x.pos;
  return r;
}
__device__ __forceinline__ TRec trec_add(const TRec& x, const TRec& y) {
  TRec r;
  r.s[0] = tside_add(x.s[0], y.s[0]);
  r.s[1] = tside_add(x.s[1], y.s[1]);
  return r;
}
__device__ __forceinline__ TRec trec_zero() {
  TRec r;
  for (int q = 0; q < 2; ++q) {
    r.s[q].g_lo = r.s[q].g_hi = r.s[q].h_lo = r.s[q].h_hi = 0ull;
    r.s[q].pos = 0; r.s[q].cnt = 0; r.s[q].val = 0.f;
  }
  return r;
}
__device__ __forceinline__ TRec trec_shfl_up(const TRec& x, int o) {
  TRec r;
  const unsigned* p = reinterpret_cast<const unsigned*>(&x);
  unsigned* d = reinterpret_cast<unsigned*>(&r);
#pragma unroll
  for (int i = 0; i < 24; ++i) d[i] = __shfl_up_sync(0xffffffffu, p[i], o);
  return r;
}
__device__ __forceinline__ TRec trec_ld(const TRec* p) {
  TRec r;
  const uint4* s = reinterpret_cast<const uint4*>(p);
  uint4* d = reinterpret_cast<uint4*>(&r);
#pragma unroll
  for (int i = 0; i < 6; ++i) d[i] = __ldcg(s + i);
  return r;
}
__device__ __forceinline__ void trec_st(TRec* p, const TRec& x) {
  const uint4* s = reinterpret_cast<const uint4*>(&x);
  uint4* d = reinterpret_cast<uint4*>(p);
#pragma unroll
  for (int i = 0; i < 6; ++i) __stcg(d + i, s[i]);
}

// largest j with off[j] <= q
__device__ __forceinline__ int seg_of(const int* off, int K, int q) {
  int lo = 0, hi = K - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (off[mid] <= q) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// exclusive block scan of an int (all threads); returns the total too
__device__ __forceinline__ int block_exscan_int(int x, int& total, int* wsum, int lane, int wid) {
  int incl = x;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += y;
  }
  if (lane == 31) wsum[wid] = incl;
  __syncthreads();
  int wex = 0, tot = 0;
#pragma unroll
  for (int w = 0; w < kFW; ++w) {
    const int s = wsum[w];
    if (w < wid) wex += s;
    tot += s;
  }
  total = tot;
  return wex + incl - x;
}

// 1/x for x > 0: hardware seed + two Newton steps (~1 ulp); ranks only (the exact Eq. 2 decides)
__device__ __forceinline__ double rcp_nr(double x) {
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
  double e = __fma_rn(-x, r, 1.0);
  r = __fma_rn(r, e, r);
  e = __fma_rn(-x, r, 1.0);
  return __fma_rn(r, e, r);
}

__device__ __forceinline__ bool rec_better_f(unsigned long long gk, const Rec& r, unsigned long long gk0, const Rec& r0) {
  return gk > gk0 || (gk == gk0 && tie_key(r.attr, r.value, r.dir) < tie_key(r0.attr, r0.value, r0.dir));
}

// ============================================================================ k_tile_agg
struct AggSmem {
  int off[kFusedMaxK + 1];
  int cidx[kFusedMaxK];
  double wg[2][2][kFW], wh[2][2][kFW];  // [tile parity][side][warp]
  int wc[2][2][kFW], wi[2][2][kFW];
};

template <int HMODE>
__global__ void __launch_bounds__(kFT) k_tile_agg(FusedArgs A) {
  __shared__ AggSmem S;
  const FusedPlan* P = A.plan;
  const int T = P->T;
  if (T == 0) return;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int K = P->K, tpa = P->tpa, n_act = (int)P->n_act;
  const long long stride = P->stride;
  const int Fg = A.fx[0], Fh = A.fx[1];
  for (int i = tid; i <= K; i += kFT) S.off[i] = P->off[i];
  for (int i = tid; i < K; i += kFT) S.cidx[i] = P->cidx[i];
  __syncthreads();
  const int qi = tid * kFI;
  int par = 0;
  for (int t = blockIdx.x; t < T; t += gridDim.x, par ^= 1) {
    const int a = t / tpa;
    const int q0 = (t - a * tpa) * kFTile;
    const int len = min(kFTile, n_act - q0);
    const long long tbase = (long long)a * stride + q0;
    const int jf = seg_of(S.off, K, q0);              // the tile's first piece
    const int jl = seg_of(S.off, K, q0 + len - 1);    // its last piece
    if ((jf != jl || !A.warp_tiles) && tid == 0) A.mlist[atomicAdd(A.mcount, 1)] = t;  // k_fused's (CTA) tiles
    const bool live_l = S.cidx[jl] >= 0;
    const int ql = S.off[jl] - q0;                    // the last piece's start, tile-relative
    int id[kFI];
    double g[kFI];
    if (qi + kFI <= len) {
      const int4 i0 = __ldcs(reinterpret_cast<const int4*>(A.ins + tbase + qi));
      const int4 i1 = __ldcs(reinterpret_cast<const int4*>(A.ins + tbase + qi) + 1);
      id[0] = i0.x; id[1] = i0.y; id[2] = i0.z; id[3] = i0.w; id[4] = i1.x; id[5] = i1.y; id[6] = i1.z; id[7] = i1.w;
      const double2* pg = reinterpret_cast<const double2*>(A.gl + tbase + qi);
#pragma unroll
      for (int k = 0; k < kFI / 2; ++k) {
        const double2 z = __ldcs(pg + k);
        g[2 * k] = z.x;
        g[2 * k + 1] = z.y;
      }
    } else {  // the list's tail: scalar loads, nothing past its end
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        const bool in = qi + k < len;
        id[k] = in ? A.ins[tbase + qi + k] : 0;
        g[k] = in ? A.gl[tbase + qi + k] : 0.0;
      }
    }
    // items whose node split (their side is looked up) and items of the last piece (summed)
    unsigned livem = 0, lastm = 0;
    const unsigned validm = qi >= len ? 0u : (qi + kFI <= len ? 0xffu : ((1u << (len - qi)) - 1u));
    if (jf == jl) {  // one segment piece: the common case
      livem = live_l ? validm : 0u;
      lastm = livem;
    } else {
      int j = seg_of(S.off, K, q0 + min(qi, len - 1));
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        while (j + 1 < K && S.off[j + 1] <= q0 + qi + k) ++j;
        if (S.cidx[j] >= 0) livem |= 1u << k;
        if (j == jl) lastm |= 1u << k;
      }
      livem &= validm;
      lastm &= livem;
    }
    unsigned w[kFI];
#pragma unroll
    for (int k = 0; k < kFI; ++k) w[k] = ((livem >> k) & 1u) ? __ldg(A.hbit + (id[k] >> 5)) : 0u;
    unsigned bits = 0;
#pragma unroll
    for (int k = 0; k < kFI; ++k) bits |= ((w[k] >> (id[k] & 31)) & 1u) << k;
    bits &= livem;
    A.tbits[(size_t)t * kFT + tid] = (unsigned char)bits;
    // the last piece's sums per side, in entry order; last entry per side
    double sg[2] = {0.0, 0.0}, sh[2] = {0.0, 0.0};
#pragma unroll
    for (int k = 0; k < kFI; ++k) {
      if ((lastm >> k) & 1u) {
        const double h = hess_of<HMODE>(g[k]);
        if ((bits >> k) & 1u) { sg[0] = sg[0] + g[k]; sh[0] = sh[0] + h; }
        else { sg[1] = sg[1] + g[k]; sh[1] = sh[1] + h; }
      }
    }
    const unsigned hm = bits & lastm, lm = ~bits & lastm;
    int sc[2] = {__popc(hm), __popc(lm)};
    int si[2] = {hm ? qi + 31 - __clz(hm) : -1, lm ? qi + 31 - __clz(lm) : -1};
    // block sums: a fixed tree (xor shuffles, then warps in order)
#pragma unroll
    for (int s = 0; s < 2; ++s) {
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        sg[s] = sg[s] + __shfl_xor_sync(0xffffffffu, sg[s], o);
        sh[s] = sh[s] + __shfl_xor_sync(0xffffffffu, sh[s], o);
        sc[s] += __shfl_xor_sync(0xffffffffu, sc[s], o);
        si[s] = max(si[s], __shfl_xor_sync(0xffffffffu, si[s], o));
      }
      if (lane == 0) {
        S.wg[par][s][wid] = sg[s]; S.wh[par][s][wid] = sh[s];
        S.wc[par][s][wid] = sc[s]; S.wi[par][s][wid] = si[s];
      }
    }
    __syncthreads();  // (the other parity's slots are free: one barrier per tile)
    if (tid < 2) {
      const int s = tid;
      double G = 0.0, H = 0.0;
      int c = 0, ix = -1;
#pragma unroll
      for (int w2 = 0; w2 < kFW; ++w2) {
        G = G + S.wg[par][s][w2]; H = H + S.wh[par][s][w2];
        c += S.wc[par][s][w2]; ix = max(ix, S.wi[par][s][w2]);
      }
      TSide r;
      const __int128 Gx = c ? to_fx(G, Fg) : 0, Hx = c ? to_fx(H, Fh) : 0;
      r.g_lo = (unsigned long long)Gx; r.g_hi = (unsigned long long)((unsigned __int128)Gx >> 64);
      r.h_lo = (unsigned long long)Hx; r.h_hi = (unsigned long long)((unsigned __int128)Hx >> 64);
      r.cnt = c;
      r.val = 0.f;  // k_fused reads the value at pos itself
      r.pos = c ? tbase + ix : 0;
      const uint4* src4 = reinterpret_cast<const uint4*>(&r);
      uint4* d4 = reinterpret_cast<uint4*>(&A.tagg[t].s[s]);
#pragma unroll
      for (int i = 0; i < 3; ++i) __stcg(d4 + i, src4[i]);
      if (s == 0) A.treset[t] = (unsigned char)(ql >= 0 || !live_l);  // the piece starts in this tile
    }
  }
}

// ============================================================================ tile scan
// S1: per group of kTSGroup tiles, the segmented inclusive scan (reset = the tile's last piece
// starts in it); the group's aggregate and whether a reset occurred up to each tile
__global__ void __launch_bounds__(kTSGroup) k_tscan1(FusedArgs A) {
  __shared__ TRec wtot[kTSGroup / 32];
  __shared__ int wf[kTSGroup / 32];
  const int T = A.plan->T;
  const int t = blockIdx.x * kTSGroup + threadIdx.x;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if ((int)(blockIdx.x * kTSGroup) >= T) return;
  TRec x = t < T ? trec_ld(A.tagg + t) : trec_zero();
  int f = t < T ? A.treset[t] : 0;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const TRec y = trec_shfl_up(x, o);
    const int yf = __shfl_up_sync(0xffffffffu, f, o);
    if (lane >= o) {
      if (!f) x = trec_add(y, x);
      f |= yf;
    }
  }
  if (lane == 31) { wtot[wid] = x; wf[wid] = f; }
  __syncthreads();
  if (!f) {
    TRec p = trec_zero();
    int pf = 0;
    for (int w = 0; w < wid; ++w) {
      p = wf[w] ? wtot[w] : trec_add(p, wtot[w]);
      pf |= wf[w];
    }
    x = trec_add(p, x);
    f = pf;
  }
  if (t < T) {
    trec_st(A.tinc + t, x);
    A.tseen[t] = (unsigned char)f;
  }
  if (threadIdx.x == kTSGroup - 1 || t == T - 1) {
    trec_st(A.tgagg + blockIdx.x, x);
    A.tgf[blockIdx.x] = (unsigned char)f;
  }
}

// S2: carries between groups: the same segmented scan over the group aggregates, one CTA, in
// chunks of kTSGroup with a running carry
__global__ void __launch_bounds__(kTSGroup) k_tscan2(FusedArgs A) {
  __shared__ TRec wtot[kTSGroup / 32];
  __shared__ int wf[kTSGroup / 32];
  __shared__ TRec run;
  const int T = A.plan->T;
  const int ng = (T + kTSGroup - 1) / kTSGroup;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  if (threadIdx.x == 0) run = trec_zero();
  __syncthreads();
  for (int b0 = 0; b0 < ng; b0 += kTSGroup) {
    const int gi = b0 + threadIdx.x;
    TRec x = gi < ng ? trec_ld(A.tgagg + gi) : trec_zero();
    int f = gi < ng ? A.tgf[gi] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const TRec y = trec_shfl_up(x, o);
      const int yf = __shfl_up_sync(0xffffffffu, f, o);
      if (lane >= o) {
        if (!f) x = trec_add(y, x);
        f |= yf;
      }
    }
    if (lane == 31) { wtot[wid] = x; wf[wid] = f; }
    __syncthreads();
    if (!f) {
      TRec p = run;
      for (int w = 0; w < wid; ++w) p = wf[w] ? wtot[w] : trec_add(p, wtot[w]);
      x = trec_add(p, x);
    }
    // exclusive: the inclusive value of the previous group
    const TRec prev = trec_shfl_up(x, 1);
    __syncthreads();
    if (gi < ng) {
      TRec ex = prev;
      if (lane == 0) {  // from the previous warp (or the previous chunk)
        TRec p = run;
        for (int w = 0; w < wid; ++w) p = wf[w] ? wtot[w] : trec_add(p, wtot[w]);
        ex = p;
      }
      trec_st(A.tgcarry + gi, ex);
    }
    __syncthreads();
    if (gi == min(ng, b0 + kTSGroup) - 1) run = x;
    __syncthreads();
  }
}

// S3: tiles before their group's first reset take the group's carry; the value of each side's
// last entry is read here once (k_fused's carry then needs no dependent load)
__global__ void __launch_bounds__(kTSGroup) k_tscan3(FusedArgs A) {
  const int T = A.plan->T;
  const int t = blockIdx.x * kTSGroup + threadIdx.x;
  if (t >= T) return;
  TRec x = trec_ld(A.tinc + t);
  if (blockIdx.x > 0 && !A.tseen[t]) x = trec_add(trec_ld(A.tgcarry + blockIdx.x), x);
  for (int q = 0; q < 2; ++q) x.s[q].val = x.s[q].cnt ? A.val[x.s[q].pos] : 0.f;
  trec_st(A.tinc + t, x);
}

// ============================================================================ k_fused
struct FusedSmem {
  float val[kFS][kFTile];
  int32_t ins[kFS][kFTile];
  double g[kFS][kFTile];
  unsigned short src[kFTile];       // child order: slot r holds tile entry src[r]
  float cval[kFTile];               // single-piece tiles: the entries moved into child order
  int32_t cins[kFTile];
  double cg[kFTile];
  int rowc[kFTile / 32];            // per 32-entry row: packed (high | low << 16) counts, then their scan
  int tot;
  unsigned long long bar[kFS];
  // plan copy
  int off[kFusedMaxK + 1];
  int cidx[kFusedMaxK];
  int offn[2 * kFusedMaxK + 1];
  double cG[2 * kFusedMaxK], cH[2 * kFusedMaxK], cHl[2 * kFusedMaxK], cP[2 * kFusedMaxK];
  // CTA node-best table (children)
  unsigned long long ngk[2 * kFusedMaxK];
  // per tile
  int j0, nseg, nk, cont;
  int pq[kFusedMaxK + 1];           // tile-relative start of piece s (pq[nseg] = tile length)
  int base[kFusedMaxK + 1];         // packed exclusive (high | low << 16) count at piece start
  int gb[2 * kFusedMaxK + 1];       // child-order group starts: group 2s = piece s high, 2s+1 low
  unsigned long long gk[2 * kFusedMaxK];
  int wr[2 * kFusedMaxK];
  int wsum[kFW];
  double wg[kFW], wh[kFW];
  int wf[kFW];
  TSide ex[2];                      // carry of the first piece (the tile scan's record of t - 1)
  double cgx[2], chx[2];            // the carry's sums as fp64 (single-piece path)
};

// rank score of a split, GL^2/(HL+l) + GR^2/(HR+l) = 2 Eq.2 + const, kept as num / den:
// candidates of a thread's run are compared by cross-multiplication (no division); the run's
// winner is then evaluated with the exact Eq. 2 expression (IEEE divisions), which alone
// decides between runs, threads, tiles and CTAs (I3)
struct Cand {
  double num, den, GL, HL;
  int r;
};

template <int HMODE, bool kWrite>
__global__ void __launch_bounds__(kFT, GBDT_FUSED_CTAS) k_fused(FusedArgs A) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  FusedSmem& S = *reinterpret_cast<FusedSmem*>(smem_raw);
  const FusedPlan* P = A.plan;
  const int T = P->T;
  if (T == 0) return;
  const int Tm = *A.mcount;  // the tiles holding several segment pieces (k_tile_agg's list)
  if (Tm == 0) return;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int K = P->K, Kn = P->Kn, tpa = P->tpa;
  const int n_act = (int)P->n_act;
  const long long stride = P->stride, stride_n = P->stride_next;
  const unsigned ep = (unsigned)P->epoch;
  const int Fg = A.fx[0], Fh = A.fx[1];
  const double lam = A.lam;
  for (int i = tid; i <= K; i += kFT) S.off[i] = P->off[i];
  for (int i = tid; i < K; i += kFT) S.cidx[i] = P->cidx[i];
  for (int i = tid; i <= Kn; i += kFT) S.offn[i] = P->offn[i];
  for (int c = tid; c < Kn; c += kFT) {
    S.cG[c] = A.nxt.G[c]; S.cH[c] = A.nxt.H[c]; S.cHl[c] = __dadd_rn(A.nxt.H[c], lam); S.cP[c] = A.nxt.pterm[c];
    S.ngk[c] = 0ull;
  }
  Rec* const nrec = A.cta_rec + (size_t)blockIdx.x * (2 * kFusedMaxK);  // CTA node-best records (global, L1)
  const unsigned long long pol = policy_evict_first();
  auto issue = [&](int st, int t) {  // TMA of tile t's lists into stage st
    const int a = t / tpa;
    const int q0 = (t - a * tpa) * kFTile;
    const long long p0 = (long long)a * stride + q0;
    const uint32_t n = (uint32_t)((min(kFTile, n_act - q0) + 3) & ~3);
    mbar_arrive_expect_tx(&S.bar[st], 16u * n);
    tma_load_1d(S.val[st], A.val + p0, 4u * n, &S.bar[st], pol);
    tma_load_1d(S.ins[st], A.ins + p0, 4u * n, &S.bar[st], pol);
    tma_load_1d(S.g[st], A.gl + p0, 8u * n, &S.bar[st], pol);
  };
  if (tid == 0) {
    for (int st = 0; st < kFS; ++st) mbar_init(&S.bar[st], 1);
    fence_mbar_init();
    for (int st = 0; st < kFS; ++st) {
      const int i = blockIdx.x + st * gridDim.x;
      if (i < Tm) issue(st, A.mlist[i]);
    }
  }
  __syncthreads();
  uint32_t phase = 0;
  const int qi = tid * kFI;
  for (int it = 0;; ++it) {
    const int ti = blockIdx.x + it * gridDim.x;
    if (ti >= Tm) break;
    const int t = A.mlist[ti];
    const int st = it % kFS;
    const int a = t / tpa;
    const int q0 = (t - a * tpa) * kFTile;
    const int len = min(kFTile, n_act - q0);
    const long long tbase = (long long)a * stride + q0;
    const float* sval = S.val[st];
    const int32_t* sins = S.ins[st];
    const double* sg = S.g[st];
    if (tid == 0) {  // the tile's pieces (parent segments), while the copy is in flight
      const int lo = seg_of(S.off, K, q0);
      int s = 0;
      S.pq[0] = 0;
      while (S.off[lo + s + 1] < q0 + len) { ++s; S.pq[s] = S.off[lo + s] - q0; }
      S.pq[s + 1] = len;
      S.j0 = lo;
      S.nseg = s + 1;
      S.cont = S.off[lo] < q0 && S.cidx[lo] >= 0;
    } else if (tid >= 32 && tid < 38) {  // carry of the first piece: the scanned record of t - 1
      const int lo = seg_of(S.off, K, q0);
      const bool c = S.off[lo] < q0 && S.cidx[lo] >= 0;
      uint4* d = reinterpret_cast<uint4*>(S.ex);
      d[tid - 32] = c ? __ldcg(reinterpret_cast<const uint4*>(A.tinc + (t - 1)) + (tid - 32)) : make_uint4(0, 0, 0, 0);
    }
    const unsigned tb = A.tbits[(size_t)t * kFT + tid];
    mbar_wait(&S.bar[st], (phase >> st) & 1);
    phase ^= 1u << st;
    __syncthreads();
    const int j0 = S.j0, nseg = S.nseg;
    const bool cont = S.cont != 0;
    bool issued = false;  // thread 0: the next tile's copy into this stage has been started

    if (nseg == 1) {
      // ================= one segment piece (the common case): two child runs, high then low.
      //  1. striped (entry k*256 + 32 w + lane): side bits per 32-entry row from k_tile_agg's
      //     words, ranks by popc, the rows' counts scanned by one warp; entries MOVED into the
      //     child-order buffer (consecutive lanes -> consecutive slots, no bank conflicts), after
      //     which the stage is free and the next tile's copy starts
      //  2. blocked (child slots 8 tid .. 8 tid + 7, 16-byte loads): segmented scans, candidates
      //  3. striped: coalesced stores of the child runs
      const int c0 = S.cidx[j0];
      if (c0 >= 0) {
        const unsigned* words = reinterpret_cast<const unsigned*>(A.tbits) + (size_t)t * (kFTile / 32);
        const unsigned myw = lane < kFI ? __ldg(words + lane * kFW + wid) : 0u;
        const unsigned ltm = (1u << lane) - 1u;
        const bool full = len == kFTile;
        unsigned wk[kFI];
#pragma unroll
        for (int k = 0; k < kFI; ++k) {
          const int e0 = k * kFT + 32 * wid;  // the row's first entry
          const unsigned vm = full ? 0xffffffffu : (e0 >= len ? 0u : (e0 + 32 <= len ? 0xffffffffu : ((1u << (len - e0)) - 1u)));
          wk[k] = __shfl_sync(0xffffffffu, myw, k) & vm;
          if (lane == 0) S.rowc[k * kFW + wid] = __popc(wk[k]) | ((__popc(vm) - __popc(wk[k])) << 16);
        }
        __syncthreads();
        if (wid == 0) {  // exclusive scan of the 64 row counts (2 per lane), in tile order
          const int x0 = S.rowc[2 * lane], x1 = S.rowc[2 * lane + 1];
          int incl = x0 + x1;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
          }
          const int exl = incl - x0 - x1;
          S.rowc[2 * lane] = exl;
          S.rowc[2 * lane + 1] = exl + x0;
          if (lane == 31) S.tot = incl;
          if (lane == 0) {
            S.gk[0] = S.gk[1] = 0ull;
            S.wr[0] = S.wr[1] = INT_MAX;
            for (int q = 0; q < 2; ++q) {  // the carries as fp64, once
              S.cgx[q] = cont ? from_fx((__int128)u128(S.ex[q].g_lo, S.ex[q].g_hi), Fg) : 0.0;
              S.chx[q] = cont ? from_fx((__int128)u128(S.ex[q].h_lo, S.ex[q].h_hi), Fh) : 0.0;
            }
          }
        }
        __syncthreads();
        const int NH = S.tot & 0xffff, NK = NH + (S.tot >> 16);
#pragma unroll
        for (int k = 0; k < kFI; ++k) {  // move into child order
          const int e = k * kFT + 32 * wid + lane;
          if (full || e < len) {
            const int b = S.rowc[k * kFW + wid];
            const bool hi = (wk[k] >> lane) & 1u;
            const int rh = __popc(wk[k] & ltm);  // high entries before this lane in the row
            const int r = hi ? (b & 0xffff) + rh : NH + (b >> 16) + (lane - rh);  // all lanes < e are valid
            S.cval[r] = sval[e];
            S.cins[r] = sins[e];
            S.cg[r] = sg[e];
            S.src[r] = (unsigned short)e;
          }
        }
        __syncthreads();
        if (tid == 0) {  // the stage is drained: start the next tile's copy now
          const int i2 = ti + kFS * gridDim.x;
          if (i2 < Tm) {
            fence_proxy_async();
            issue(st, A.mlist[i2]);
          }
          issued = true;
        }
        // child-order slots r = qi .. qi + 7: high run [0, NH), low run [NH, NK); heads at 0, NH
        double gv[kFI], hv[kFI];
        float vv[kFI];
        {
          const double2* pg = reinterpret_cast<const double2*>(S.cg + qi);
          const float4* pv = reinterpret_cast<const float4*>(S.cval + qi);
#pragma unroll
          for (int k = 0; k < kFI / 2; ++k) {
            const double2 z = pg[k];
            gv[2 * k] = z.x;
            gv[2 * k + 1] = z.y;
          }
          const float4 a0 = pv[0], a1 = pv[1];
          vv[0] = a0.x; vv[1] = a0.y; vv[2] = a0.z; vv[3] = a0.w; vv[4] = a1.x; vv[5] = a1.y; vv[6] = a1.z; vv[7] = a1.w;
        }
        const int kh = NH - qi;  // item index of slot NH in this thread, if 0 <= kh < kFI
        const unsigned headm = (qi == 0 ? 1u : 0u) | ((kh >= 0 && kh < kFI && NH < NK) ? (1u << kh) : 0u);
        const int nin = min(kFI, NK - qi);  // slots of this thread (may be <= 0)
        double ag = 0.0, ah = 0.0;
#pragma unroll
        for (int k = 0; k < kFI; ++k) {
          hv[k] = hess_of<HMODE>(gv[k]);
          if (k < nin) {
            if ((headm >> k) & 1u) { ag = gv[k]; ah = hv[k]; }
            else { ag = ag + gv[k]; ah = ah + hv[k]; }
          }
        }
        double ig = ag, ih = ah;
        int iflag = headm != 0u;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const double yg = __shfl_up_sync(0xffffffffu, ig, o), yh = __shfl_up_sync(0xffffffffu, ih, o);
          const int yf = __shfl_up_sync(0xffffffffu, iflag, o);
          if (lane >= o) {
            if (!iflag) { ig = yg + ig; ih = yh + ih; }
            iflag |= yf;
          }
        }
        if (lane == 31) { S.wg[wid] = ig; S.wh[wid] = ih; S.wf[wid] = iflag; }
        double eg = __shfl_up_sync(0xffffffffu, ig, 1), eh = __shfl_up_sync(0xffffffffu, ih, 1);
        int ef = __shfl_up_sync(0xffffffffu, iflag, 1);
        if (lane == 0) { eg = 0.0; eh = 0.0; ef = 0; }
        __syncthreads();
        if (!ef) {
          double pg = 0.0, ph = 0.0;
          for (int w = 0; w < wid; ++w) {
            if (S.wf[w]) { pg = S.wg[w]; ph = S.wh[w]; }
            else { pg = pg + S.wg[w]; ph = ph + S.wh[w]; }
          }
          eg = pg + eg;
          eh = ph + eh;
        }
        // GL, HL of a slot = carry of its run + the tile's sum over the run's earlier slots,
        // associated as (carry + eg) + g_k ... (fixed, so ranking and record agree)
        const int q0s = qi < NH ? 0 : 1;  // run of the thread's first slot
        const double sg0 = S.cgx[q0s] + eg, sh0 = S.chx[q0s] + eh;
        int ra_g = -1, rb_g = -1, ra_r = -1, rb_r = -1;
        unsigned long long ra_k = 0ull, rb_k = 0ull;
        double aGL = 0, aHL = 0, bGL = 0, bHL = 0;
        if (nin > 0) {
          int q = q0s;
          int c = c0 + q;
          double Gc = S.cG[c], Hl = S.cHl[c];
          double rg = sg0, rh = sh0;
          double bnum = -1.0, bden = 1.0, bGLc = 0.0, bHLc = 0.0;
          int br = -1;
          float pv;
          bool prev;
          if (qi != 0 && qi != NH) { pv = S.cval[qi - 1]; prev = true; }
          else { prev = cont && S.ex[q].cnt > 0; pv = S.ex[q].val; }
#pragma unroll
          for (int k = 0; k < kFI; ++k) {
            if (k < nin) {
              const int r = qi + k;
              if ((headm >> k) & 1u) {
                if (k > 0) {  // the low run starts inside this thread: close the high one
                  if (br >= 0) { ra_g = 0; ra_r = br; aGL = bGLc; aHL = bHLc; }
                  q = 1; c = c0 + 1; Gc = S.cG[c]; Hl = S.cHl[c];
                  bnum = -1.0; bden = 1.0; br = -1;
                  prev = cont && S.ex[1].cnt > 0;
                  pv = S.ex[1].val;
                }
                rg = S.cgx[q];
                rh = S.chx[q];
              }
              const float cv = vv[k];
              if (prev && pv != cv) {
                const double dl = rh + lam, dr = Hl - rh, GR = Gc - rg;
                const double num = __fma_rn(rg * rg, dr, (GR * GR) * dl), den = dl * dr;
                if (num * bden > bnum * den) { bnum = num; bden = den; br = r; bGLc = rg; bHLc = rh; }
              }
              rg = rg + gv[k];
              rh = rh + hv[k];
              pv = cv;
              prev = true;
            }
          }
          if (br >= 0) {
            if (ra_g < 0 && !(q == 1 && qi < NH)) { ra_g = q; ra_r = br; aGL = bGLc; aHL = bHLc; }
            else { rb_g = q; rb_r = br; bGL = bGLc; bHL = bHLc; }
          }
        }
        if (ra_g >= 0) { const int c = c0 + ra_g; ra_k = gain_key(eq2_gain(aGL, aHL, S.cG[c], S.cH[c], lam, S.cP[c])); }
        if (rb_g >= 0) { const int c = c0 + rb_g; rb_k = gain_key(eq2_gain(bGL, bHL, S.cG[c], S.cH[c], lam, S.cP[c])); }
        {  // group maxima: the first run through a warp reduction, the other one directly
          const unsigned peers = __match_any_sync(0xffffffffu, ra_g);
          const unsigned hi = __reduce_max_sync(peers, (unsigned)(ra_k >> 32));
          const unsigned lo = __reduce_max_sync(peers, (unsigned)(ra_k >> 32) == hi ? (unsigned)ra_k : 0u);
          if (ra_g >= 0 && lane == __ffs(peers) - 1) atomicMax(&S.gk[ra_g], ((unsigned long long)hi << 32) | lo);
          if (rb_g >= 0) atomicMax(&S.gk[rb_g], rb_k);
        }
        __syncthreads();
        if (ra_g >= 0 && ra_k == S.gk[ra_g]) atomicMin(&S.wr[ra_g], ra_r);  // ties: the larger value
        if (rb_g >= 0 && rb_k == S.gk[rb_g]) atomicMin(&S.wr[rb_g], rb_r);
        __syncthreads();
#pragma unroll
        for (int i = 0; i < 2; ++i) {
          const int gq = i ? rb_g : ra_g, r = i ? rb_r : ra_r;
          const unsigned long long key = i ? rb_k : ra_k;
          if (gq < 0 || S.wr[gq] != r || key != S.gk[gq]) continue;
          const int gs = gq ? NH : 0;
          const int c = c0 + gq;
          Rec rc;
          rc.GL = i ? bGL : aGL;
          rc.HL = i ? bHL : aHL;
          rc.cntL = (cont ? S.ex[gq].cnt : 0) + (r - gs);
          rc.gain = eq2_gain(rc.GL, rc.HL, S.cG[c], S.cH[c], lam, S.cP[c]);
          rc.value = r > gs ? S.cval[r - 1] : S.ex[gq].val;
          rc.pos = r > gs ? tbase + S.src[r - 1] : S.ex[gq].pos;
          rc.attr = A.a_base + a;
          rc.dir = 0;
          rc.node = c;
          rc.epoch = (int)ep;
          rc.shard = A.shard;
          if (rec_better_f(key, rc, S.ngk[c], nrec[c])) {  // one writer per child node per tile
            nrec[c] = rc;
            S.ngk[c] = key;
          }
        }
        if (kWrite) {  // child runs -> the next level's lists, 32 consecutive slots per warp
          const long long bh = (long long)a * stride_n + S.offn[c0] + (cont ? S.ex[0].cnt : 0);
          const long long bl = (long long)a * stride_n + S.offn[c0 + 1] + (cont ? S.ex[1].cnt : 0) - NH;
          for (int r = tid; r < NK; r += kFT) {
            const long long d = (r < NH ? bh : bl) + r;
            __stcs(A.val_out + d, S.cval[r]);
            __stcs(A.ins_out + d, S.cins[r]);
            __stcs(A.g_out + d, S.cg[r]);
          }
        }
      }
    } else {
#ifndef GBDT_FUSED_NO_GENERAL
    // ---- 1. stable in-tile partition by (piece, side) -> src[]
    int sidx[kFI];  // piece << 2 | side (1 high, 2 low); -1 dropped
    {
      int s = 0;
      while (s + 1 < nseg && qi >= S.pq[s + 1]) ++s;
      int nb = S.pq[s + 1];
      bool live = S.cidx[j0 + s] >= 0;
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        if (qi + k >= nb && s + 1 < nseg) {
          ++s;
          nb = S.pq[s + 1];
          live = S.cidx[j0 + s] >= 0;
        }
        sidx[k] = (qi + k < len && live) ? ((s << 2) | (((tb >> k) & 1u) ? 1 : 2)) : -1;
      }
    }
    int pc = 0;
#pragma unroll
    for (int k = 0; k < kFI; ++k) pc += sidx[k] < 0 ? 0 : ((sidx[k] & 1) ? 1 : (1 << 16));
    int tot;
    const int ex = block_exscan_int(pc, tot, S.wsum, lane, wid);
    if (nseg > 1) {  // packed count at every piece start (the thread holding the start writes it)
      int e = ex;
      int z = 1;
      while (z < nseg && S.pq[z] < qi) ++z;
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        if (z < nseg && S.pq[z] == qi + k) { S.base[z] = e; ++z; }
        e += sidx[k] < 0 ? 0 : ((sidx[k] & 1) ? 1 : (1 << 16));
      }
    }
    if (tid == 0) { S.base[0] = 0; S.base[nseg] = tot; }
    for (int i = tid; i < 2 * nseg; i += kFT) { S.gk[i] = 0ull; S.wr[i] = INT_MAX; }
    __syncthreads();
    if (tid <= nseg) {
      const int b = S.base[tid];
      const int R = (b & 0xffff) + (b >> 16);
      if (tid < nseg) {
        S.gb[2 * tid] = R;
        S.gb[2 * tid + 1] = R + (S.base[tid + 1] & 0xffff) - (b & 0xffff);
      } else {
        S.gb[2 * nseg] = R;
        S.nk = R;
      }
    }
    __syncthreads();
    {
      int e = ex;
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        if (sidx[k] >= 0) {
          const int s = sidx[k] >> 2;
          const int b = S.base[s];
          const int r = (sidx[k] & 1) ? S.gb[2 * s] + ((e & 0xffff) - (b & 0xffff))
                                      : S.gb[2 * s + 1] + ((e >> 16) - (b >> 16));
          S.src[r] = (unsigned short)(qi + k);
          e += (sidx[k] & 1) ? 1 : (1 << 16);
        }
      }
    }
    __syncthreads();
    const int nk = S.nk;

    // ---- 2. segmented prefix sums over the child runs (child-order slots r = qi .. qi + 7)
    int grp0 = 0;
    {
      const int r0 = min(qi, max(nk - 1, 0));
      while (grp0 + 1 < 2 * nseg && r0 >= S.gb[grp0 + 1]) ++grp0;
    }
    double xg[kFI], xh[kFI];
    unsigned headm = 0, gstep = 0;  // gstep bit k: item k lies in a later group than item k-1
    int sr[kFI];
    {
      const uint4 sv = reinterpret_cast<const uint4*>(S.src + qi)[0];
      sr[0] = sv.x & 0xffff; sr[1] = sv.x >> 16; sr[2] = sv.y & 0xffff; sr[3] = sv.y >> 16;
      sr[4] = sv.z & 0xffff; sr[5] = sv.z >> 16; sr[6] = sv.w & 0xffff; sr[7] = sv.w >> 16;
      int gg = grp0, gn = S.gb[grp0 + 1];
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        const int r = qi + k;
        xg[k] = 0.0;
        xh[k] = 0.0;
        if (r < nk) {
          if (r >= gn) {
            while (r >= gn) { ++gg; gn = S.gb[gg + 1]; }
            if (k) gstep |= 1u << k;
          }
          if (r == S.gb[gg]) headm |= 1u << k;
          xg[k] = sg[sr[k]];
          xh[k] = hess_of<HMODE>(xg[k]);
        }
      }
    }
    // thread aggregate since its last head; warp / block segmented exclusive scans
    double ag = 0.0, ah = 0.0;
#pragma unroll
    for (int k = 0; k < kFI; ++k) {
      if ((headm >> k) & 1u) { ag = xg[k]; ah = xh[k]; }
      else { ag = ag + xg[k]; ah = ah + xh[k]; }
    }
    double ig = ag, ih = ah;
    int iflag = headm != 0u;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const double yg = __shfl_up_sync(0xffffffffu, ig, o), yh = __shfl_up_sync(0xffffffffu, ih, o);
      const int yf = __shfl_up_sync(0xffffffffu, iflag, o);
      if (lane >= o) {
        if (!iflag) { ig = yg + ig; ih = yh + ih; }
        iflag |= yf;
      }
    }
    if (lane == 31) { S.wg[wid] = ig; S.wh[wid] = ih; S.wf[wid] = iflag; }
    double eg = __shfl_up_sync(0xffffffffu, ig, 1), eh = __shfl_up_sync(0xffffffffu, ih, 1);
    int ef = __shfl_up_sync(0xffffffffu, iflag, 1);
    if (lane == 0) { eg = 0.0; eh = 0.0; ef = 0; }
    __syncthreads();
    if (!ef) {  // the prefix reaches into earlier warps: their segmented total first
      double pg = 0.0, ph = 0.0;
      for (int w = 0; w < wid; ++w) {
        if (S.wf[w]) { pg = S.wg[w]; ph = S.wh[w]; }
        else { pg = pg + S.wg[w]; ph = ph + S.wh[w]; }
      }
      eg = pg + eg;
      eh = ph + eh;
    }
    {  // exclusive in-tile prefix per slot (replaces g, h)
      double rg = eg, rh = eh;
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        if ((headm >> k) & 1u) { rg = 0.0; rh = 0.0; }
        const double ng_ = rg + xg[k], nh_ = rh + xh[k];
        xg[k] = rg;
        xh[k] = rh;
        rg = ng_;
        rh = nh_;
      }
    }

    // ---- 3. candidates: the boundary before every child entry whose predecessor in its child
    // segment has another value (the predecessor ends a run); GL, HL = sums over the
    // predecessor and everything before it.  Per run of the thread's slots in one group: the
    // best by score, then its exact Eq. 2 gain.
    double cgx[2] = {0.0, 0.0}, chx[2] = {0.0, 0.0};
    if (cont) {
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        cgx[q] = from_fx((__int128)u128(S.ex[q].g_lo, S.ex[q].g_hi), Fg);
        chx[q] = from_fx((__int128)u128(S.ex[q].h_lo, S.ex[q].h_hi), Fh);
      }
    }
    // runs of this thread: (group, key, slot, GL, HL); closed at group changes (local memory)
    int nrun = 0;
    int rgrp[kFI], rslot[kFI];
    unsigned long long rkey[kFI];
    double rGL[kFI], rHL[kFI];
    if (qi < nk) {
      int gg = grp0;
      int gs = S.gb[gg];
      int q = gg & 1;
      int c = S.cidx[j0 + (gg >> 1)] + q;
      bool carry = (gg >> 1) == 0 && cont;
      double Gc = S.cG[c], Hl = S.cHl[c];
      Cand b{-1.0, 1.0, 0.0, 0.0, -1};
      float pv;
      bool prev;
      if (qi > gs) { pv = sval[S.src[qi - 1]]; prev = true; }
      else { prev = carry && S.ex[q].cnt > 0; pv = S.ex[q].val; }
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        const int r = qi + k;
        if (r < nk) {
          if ((gstep >> k) & 1u) {  // a later group starts here: close the run
            if (b.r >= 0) {
              rgrp[nrun] = gg; rslot[nrun] = b.r; rGL[nrun] = b.GL; rHL[nrun] = b.HL;
              rkey[nrun] = gain_key(eq2_gain(b.GL, b.HL, Gc, S.cH[c], lam, S.cP[c]));
              ++nrun;
            }
            while (r >= S.gb[gg + 1]) ++gg;
            gs = S.gb[gg];
            q = gg & 1;
            c = S.cidx[j0 + (gg >> 1)] + q;
            carry = (gg >> 1) == 0 && cont;
            Gc = S.cG[c];
            Hl = S.cHl[c];
            b = Cand{-1.0, 1.0, 0.0, 0.0, -1};
            // r is its group's first slot: its predecessor, if any, is the carry's last entry
            prev = carry && S.ex[q].cnt > 0;
            pv = S.ex[q].val;
          }
          const float cv = sval[sr[k]];
          if (prev && pv != cv) {
            const double GL = carry ? __dadd_rn(q ? cgx[1] : cgx[0], xg[k]) : xg[k];
            const double HL = carry ? __dadd_rn(q ? chx[1] : chx[0], xh[k]) : xh[k];
            const double dl = HL + lam, dr = Hl - HL, GR = Gc - GL;
            const double num = __fma_rn(GL * GL, dr, (GR * GR) * dl), den = dl * dr;
            if (num * b.den > b.num * den) b = Cand{num, den, GL, HL, r};
          }
          pv = cv;
          prev = true;
        }
      }
      if (b.r >= 0) {
        rgrp[nrun] = gg; rslot[nrun] = b.r; rGL[nrun] = b.GL; rHL[nrun] = b.HL;
        rkey[nrun] = gain_key(eq2_gain(b.GL, b.HL, Gc, S.cH[c], lam, S.cP[c]));
        ++nrun;
      }
    }
    // group maxima: the thread's first run through a warp reduction over the lanes sharing its
    // group (64-bit shared atomicMax is a CAS loop), its later runs straight to shared memory
    {
      const int g1 = nrun ? rgrp[0] : -1;
      const unsigned long long k1 = nrun ? rkey[0] : 0ull;
      const unsigned peers = __match_any_sync(0xffffffffu, g1);
      const unsigned hi = __reduce_max_sync(peers, (unsigned)(k1 >> 32));
      const unsigned lo = __reduce_max_sync(peers, (unsigned)(k1 >> 32) == hi ? (unsigned)k1 : 0u);
      if (g1 >= 0 && lane == __ffs(peers) - 1) atomicMax(&S.gk[g1], ((unsigned long long)hi << 32) | lo);
      for (int i = 1; i < nrun; ++i) atomicMax(&S.gk[rgrp[i]], rkey[i]);
    }
    __syncthreads();
    for (int i = 0; i < nrun; ++i)
      if (rkey[i] == S.gk[rgrp[i]]) atomicMin(&S.wr[rgrp[i]], rslot[i]);  // ties: the larger value
    __syncthreads();
    for (int i = 0; i < nrun; ++i) {
      const int gg = rgrp[i], r = rslot[i];
      if (S.wr[gg] != r || rkey[i] != S.gk[gg]) continue;
      const int s = gg >> 1, q = gg & 1;
      const int gs = S.gb[gg];
      const int c = S.cidx[j0 + s] + q;
      const bool carry = s == 0 && cont;
      Rec rc;
      rc.GL = rGL[i];
      rc.HL = rHL[i];
      rc.cntL = (carry ? S.ex[q].cnt : 0) + (r - gs);
      rc.gain = eq2_gain(rc.GL, rc.HL, S.cG[c], S.cH[c], lam, S.cP[c]);
      const int ps = r > gs ? S.src[r - 1] : -1;
      rc.value = ps >= 0 ? sval[ps] : S.ex[q].val;
      rc.pos = ps >= 0 ? tbase + ps : S.ex[q].pos;
      rc.attr = A.a_base + a;
      rc.dir = 0;
      rc.node = c;
      rc.epoch = (int)ep;
      rc.shard = A.shard;
      if (rec_better_f(rkey[i], rc, S.ngk[c], nrec[c])) {  // one writer per child node per tile
        nrec[c] = rc;
        S.ngk[c] = rkey[i];
      }
    }
    // ---- 4. child runs -> the next level's lists (coalesced: 32 consecutive slots per warp)
    if (kWrite) {
      int gg = 0, gn = -1;
      long long dbase = 0;
      for (int r = tid; r < nk; r += kFT) {
        if (r >= gn) {
          while (r >= S.gb[gg + 1]) ++gg;
          gn = S.gb[gg + 1];
          const int s = gg >> 1, q = gg & 1;
          dbase = (long long)a * stride_n + S.offn[S.cidx[j0 + s] + q] + ((s == 0 && cont) ? S.ex[q].cnt : 0) -
                  S.gb[gg];
        }
        const int e = S.src[r];
        __stcs(A.val_out + dbase + r, sval[e]);
        __stcs(A.ins_out + dbase + r, sins[e]);
        __stcs(A.g_out + dbase + r, sg[e]);
      }
    }
#endif
    }  // general path
    __syncthreads();  // stage st and the tile scratch are free
    if (tid == 0 && !issued) {
      const int i2 = ti + kFS * gridDim.x;
      if (i2 < Tm) {
        fence_proxy_async();
        issue(st, A.mlist[i2]);
      }
    }
  }
  __syncthreads();
  // flush the CTA's node bests (R12 merge across CTAs by k_pick_tie / k_pick_best)
  for (int c = tid; c < Kn; c += kFT) {
    if (S.ngk[c]) {
      const int gs = atomicAdd(A.nrec, 1);
      A.rec[gs] = nrec[c];
      atomicMax(A.gkey + c, S.ngk[c]);
    }
  }
}

// ============================================================================ k_fusedw
// Warp-granular pass over the single-piece tiles (the common case: one parent segment per tile).
// One warp owns a 2048-entry tile end to end and streams it as eight 256-entry chunks through a
// per-warp 2-stage TMA ring; no CTA barrier anywhere.  Per chunk:
//   blocked  (lane l: entries 8 l .. 8 l + 7): sides from k_tile_agg's byte, the per-side sums of
//            the lane, one warp scan of (g_hi, h_hi, g_lo, h_lo), the lane's run ends of each
//            child run, ranked by cross-multiplied scores; the chunk's best per side by integer
//            reductions on the score bits, its exact Eq. 2 gain against the tile's best
//   striped  (row r, lane l: entry 32 r + l): coalesced stores of the child runs, ranks by popc of
//            the row's side word
// The carry between chunks stays in registers; the tile's first carry is the tile scan's record.
#ifndef GBDT_FUSEDW_CTAS
#define GBDT_FUSEDW_CTAS 2
#endif
constexpr int kWCh = 256;   // entries per chunk
constexpr int kWW = 8;      // warps per CTA
struct __align__(16) WStage {
  float val[kWCh];
  int32_t ins[kWCh];
  double g[kWCh];
};
struct __align__(16) WWarp {
  WStage st[2];
  unsigned long long bar[2];
};
struct WSmem {
  WWarp w[kWW];
  int off[kFusedMaxK + 1];
  int cidx[kFusedMaxK];
  int offn[2 * kFusedMaxK + 1];
  double cG[2 * kFusedMaxK], cH[2 * kFusedMaxK], cP[2 * kFusedMaxK];
};

// order-preserving u64 of a score >= 0 or -inf (no NaN)
__device__ __forceinline__ unsigned long long score_key(double x) {
  unsigned long long b = (unsigned long long)__double_as_longlong(x);
  return (b >> 63) ? ~b : (b | 0x8000000000000000ull);
}
__device__ __forceinline__ unsigned long long warp_max_u64(unsigned long long k) {
  const unsigned hi = __reduce_max_sync(0xffffffffu, (unsigned)(k >> 32));
  const unsigned lo = __reduce_max_sync(0xffffffffu, (unsigned)(k >> 32) == hi ? (unsigned)k : 0u);
  return ((unsigned long long)hi << 32) | lo;
}

template <int HMODE, bool kWrite>
__global__ void __launch_bounds__(kWW * 32, GBDT_FUSEDW_CTAS) k_fusedw(FusedArgs A) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  WSmem& S = *reinterpret_cast<WSmem*>(smem_raw);
  const FusedPlan* P = A.plan;
  const int T = P->T;
  if (T == 0) return;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int K = P->K, Kn = P->Kn, tpa = P->tpa;
  const int n_act = (int)P->n_act;
  const long long stride = P->stride, stride_n = P->stride_next;
  const unsigned ep = (unsigned)P->epoch;
  const int Fg = A.fx[0], Fh = A.fx[1];
  const double lam = A.lam;
  for (int i = threadIdx.x; i <= K; i += blockDim.x) S.off[i] = P->off[i];
  for (int i = threadIdx.x; i < K; i += blockDim.x) S.cidx[i] = P->cidx[i];
  for (int i = threadIdx.x; i <= Kn; i += blockDim.x) S.offn[i] = P->offn[i];
  for (int c = threadIdx.x; c < Kn; c += blockDim.x) { S.cG[c] = A.nxt.G[c]; S.cH[c] = A.nxt.H[c]; S.cP[c] = A.nxt.pterm[c]; }
  WWarp& W = S.w[wid];
  if (lane == 0) {
    mbar_init(&W.bar[0], 1);
    mbar_init(&W.bar[1], 1);
    fence_mbar_init();
  }
  __syncthreads();  // the only CTA barrier: tables and barriers are ready
  const unsigned long long pol = policy_evict_first();
  const unsigned ltm = (1u << lane) - 1u;
  uint32_t ph = 0;
  for (int t = blockIdx.x * kWW + wid; t < T; t += gridDim.x * kWW) {
    const int a = t / tpa;
    const int q0 = (t - a * tpa) * kFTile;
    const int len = min(kFTile, n_act - q0);
    const int j0 = seg_of(S.off, K, q0);
    if (S.off[j0 + 1] < q0 + len) continue;  // several pieces: k_fused's
    const int c0 = S.cidx[j0];
    if (c0 < 0) continue;                    // the node became a leaf: entries dropped
    const bool cont = S.off[j0] < q0;
    const long long tbase = (long long)a * stride + q0;
    const int nch = (len + kWCh - 1) / kWCh;
    auto issue = [&](int ch) {
      if (lane == 0 && ch < nch) {
        const int st = ch & 1;
        const long long p0 = tbase + (long long)ch * kWCh;
        const uint32_t n = (uint32_t)((min(kWCh, len - ch * kWCh) + 3) & ~3);
        fence_proxy_async();
        mbar_arrive_expect_tx(&W.bar[st], 16u * n);
        tma_load_1d(W.st[st].val, A.val + p0, 4u * n, &W.bar[st], pol);
        tma_load_1d(W.st[st].ins, A.ins + p0, 4u * n, &W.bar[st], pol);
        tma_load_1d(W.st[st].g, A.gl + p0, 8u * n, &W.bar[st], pol);
      }
    };
    issue(0);
    issue(1);
    // carry per side (0 high, 1 low): entries, sums, last value / position (warp-uniform)
    int ccnt[2] = {0, 0};
    double cg[2] = {0.0, 0.0}, chh[2] = {0.0, 0.0};
    float cv[2] = {0.f, 0.f};
    long long cpos[2] = {0, 0};
    if (cont) {
      const TRec* pr = A.tinc + (t - 1);
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const TSide x = pr->s[q];
        ccnt[q] = x.cnt;
        cg[q] = from_fx((__int128)u128(x.g_lo, x.g_hi), Fg);
        chh[q] = from_fx((__int128)u128(x.h_lo, x.h_hi), Fh);
        cv[q] = x.val;
        cpos[q] = x.pos;
      }
    }
    double Gc[2], Hc[2], Hl[2], Pc[2];
#pragma unroll
    for (int q = 0; q < 2; ++q) { Gc[q] = S.cG[c0 + q]; Hc[q] = S.cH[c0 + q]; Hl[q] = Hc[q] + lam; Pc[q] = S.cP[c0 + q]; }
    // the tile's best per side (warp-uniform): exact gain key, then the R12 tie (larger value)
    unsigned long long bkey[2] = {0ull, 0ull};
    double bGL[2] = {0, 0}, bHL[2] = {0, 0};
    long long bcnt[2] = {0, 0}, bpos[2] = {0, 0};
    float bval[2] = {0.f, 0.f};
    const long long dbase0 = (long long)a * stride_n + S.offn[c0];
    const long long dbase1 = (long long)a * stride_n + S.offn[c0 + 1];
    const unsigned char* tb = A.tbits + (size_t)t * kFT;
    for (int ch = 0; ch < nch; ++ch) {
      const int st = ch & 1;
      const int clen = min(kWCh, len - ch * kWCh);
      const unsigned hb_raw = tb[ch * 32 + lane];
      mbar_wait(&W.bar[st], (ph >> st) & 1);
      ph ^= 1u << st;
      const WStage& SG = W.st[st];
      const int k0 = lane * 8;
      const unsigned vm = k0 >= clen ? 0u : (k0 + 8 <= clen ? 0xffu : ((1u << (clen - k0)) - 1u));
      const unsigned hm = hb_raw & vm, lm = ~hb_raw & vm;
      double g[8];
      float v[8];
      {
        const double2* pg = reinterpret_cast<const double2*>(SG.g + k0);
        const float4* pv = reinterpret_cast<const float4*>(SG.val + k0);
#pragma unroll
        for (int k = 0; k < 4; ++k) { const double2 z = pg[k]; g[2 * k] = z.x; g[2 * k + 1] = z.y; }
        const float4 a0 = pv[0], a1 = pv[1];
        v[0] = a0.x; v[1] = a0.y; v[2] = a0.z; v[3] = a0.w; v[4] = a1.x; v[5] = a1.y; v[6] = a1.z; v[7] = a1.w;
      }
      // lane sums per side, in item order
      double lg[2] = {0.0, 0.0}, lh[2] = {0.0, 0.0};
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        if ((vm >> k) & 1u) {
          const double h = hess_of<HMODE>(g[k]);
          if ((hm >> k) & 1u) { lg[0] = lg[0] + g[k]; lh[0] = lh[0] + h; }
          else { lg[1] = lg[1] + g[k]; lh[1] = lh[1] + h; }
        }
      }
      // warp scans: inclusive (g, h) per side and the packed counts
      double ig[2] = {lg[0], lg[1]}, ih[2] = {lh[0], lh[1]};
      int icnt = __popc(hm) | (__popc(lm) << 16);
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
#pragma unroll
        for (int q = 0; q < 2; ++q) {
          const double yg = __shfl_up_sync(0xffffffffu, ig[q], o), yh = __shfl_up_sync(0xffffffffu, ih[q], o);
          if (lane >= o) { ig[q] = yg + ig[q]; ih[q] = yh + ih[q]; }
        }
        const int yc = __shfl_up_sync(0xffffffffu, icnt, o);
        if (lane >= o) icnt += yc;
      }
      const int excnt = icnt - (__popc(hm) | (__popc(lm) << 16));
      const int totc = __shfl_sync(0xffffffffu, icnt, 31);
      // the lane's exclusive prefix per side: carry + (exclusive in-chunk) -- (carry + eg) + items
      double rg[2], rh[2];
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        double eg = __shfl_up_sync(0xffffffffu, ig[q], 1), eh = __shfl_up_sync(0xffffffffu, ih[q], 1);
        if (lane == 0) { eg = 0.0; eh = 0.0; }
        rg[q] = cg[q] + eg;
        rh[q] = chh[q] + eh;
      }
      // the last same-side value before the lane's first item of that side
      float pv[2];
      bool prev[2];
      int pidx[2];  // chunk index of that entry (or -1: the carry's)
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const unsigned m = q ? lm : hm;
        const unsigned has = __ballot_sync(0xffffffffu, m != 0u);
        const int lastk = m ? 31 - __clz(m) : 0;
        const float lastv = v[lastk];
        const unsigned below = has & ltm;
        const int src = below ? 31 - __clz(below) : 0;
        const float sv = __shfl_sync(0xffffffffu, lastv, src);
        const int sk = __shfl_sync(0xffffffffu, k0 + lastk, src);  // the source lane's own index
        prev[q] = below ? true : ccnt[q] > 0;
        pv[q] = below ? sv : cv[q];
        pidx[q] = below ? sk : -1;
      }
      // candidates: the boundary before each item whose predecessor on its side has another value
      double bnum[2] = {-1.0, -1.0}, bden[2] = {1.0, 1.0};
      int bk[2] = {-1, -1}, bpk[2] = {-1, -1};  // winning item, its predecessor's chunk index
      double wGL[2] = {0, 0}, wHL[2] = {0, 0};
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        if ((vm >> k) & 1u) {
          const int q = ((hm >> k) & 1u) ? 0 : 1;
          const double GL = q ? rg[1] : rg[0], HL = q ? rh[1] : rh[0];
          const bool pq = q ? prev[1] : prev[0];
          const float pvq = q ? pv[1] : pv[0];
          if (pq && pvq != v[k]) {
            const double H_l = q ? Hl[1] : Hl[0], G_c = q ? Gc[1] : Gc[0];
            const double dl = HL + lam, dr = H_l - HL, GR = G_c - GL;
            const double num = __fma_rn(GL * GL, dr, (GR * GR) * dl), den = dl * dr;
            const double on = q ? bnum[1] : bnum[0], od = q ? bden[1] : bden[0];
            if (num * od > on * den) {
              if (q) { bnum[1] = num; bden[1] = den; bk[1] = k; wGL[1] = GL; wHL[1] = HL; bpk[1] = q ? pidx[1] : pidx[0]; }
              else { bnum[0] = num; bden[0] = den; bk[0] = k; wGL[0] = GL; wHL[0] = HL; bpk[0] = pidx[0]; }
            }
          }
          const double h = hess_of<HMODE>(g[k]);
          if (q) { rg[1] = rg[1] + g[k]; rh[1] = rh[1] + h; pv[1] = v[k]; prev[1] = true; pidx[1] = k0 + k; }
          else { rg[0] = rg[0] + g[k]; rh[0] = rh[0] + h; pv[0] = v[k]; prev[0] = true; pidx[0] = k0 + k; }
        }
      }
      // the chunk's best per side: approximate score max, then the smallest item (larger value)
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const double sc = bk[q] >= 0 ? bnum[q] * rcp_nr(bden[q]) : -INFINITY;
        const unsigned long long key = warp_max_u64(score_key(sc));
        if (key == score_key(-INFINITY)) continue;  // no candidate on this side in the chunk
        const unsigned idx = __reduce_min_sync(0xffffffffu, (score_key(sc) == key && bk[q] >= 0) ? (unsigned)(k0 + bk[q]) : 0xffffffffu);
        const int wl = (int)(idx >> 3);
        double GL = __shfl_sync(0xffffffffu, wGL[q], wl), HL = __shfl_sync(0xffffffffu, wHL[q], wl);
        const int pk = __shfl_sync(0xffffffffu, bpk[q], wl);
        const unsigned long long gk = gain_key(eq2_gain(GL, HL, Gc[q], Hc[q], lam, Pc[q]));
        // side counts before the winner: carry + same-side entries of the chunk before it
        const int before_lane = q ? (__shfl_sync(0xffffffffu, excnt, wl) >> 16) : (__shfl_sync(0xffffffffu, excnt, wl) & 0xffff);
        const unsigned wm = __shfl_sync(0xffffffffu, q ? lm : hm, wl);
        const long long cntL = ccnt[q] + before_lane + __popc(wm & ((1u << (idx & 7)) - 1u));
        const float pval = pk >= 0 ? SG.val[pk] : cv[q];
        const long long ppos = pk >= 0 ? tbase + (long long)ch * kWCh + pk : cpos[q];
        // R12 inside the tile: larger gain, then the larger value (the earlier candidate)
        if (gk > bkey[q]) {
          bkey[q] = gk; bGL[q] = GL; bHL[q] = HL; bcnt[q] = cntL; bval[q] = pval; bpos[q] = ppos;
        }
      }
      // carry update per side (warp-uniform)
      const int th = totc & 0xffff, tl = totc >> 16;
#pragma unroll
      for (int q = 0; q < 2; ++q) {
        const double tg = __shfl_sync(0xffffffffu, ig[q], 31), thh = __shfl_sync(0xffffffffu, ih[q], 31);
        cg[q] = cg[q] + tg;
        chh[q] = chh[q] + thh;
        const unsigned m = q ? lm : hm;
        const unsigned has = __ballot_sync(0xffffffffu, m != 0u);
        if (has) {
          const int src = 31 - __clz(has);
          const int lastk = m ? 31 - __clz(m) : 0;
          cv[q] = __shfl_sync(0xffffffffu, v[lastk], src);
          cpos[q] = tbase + (long long)ch * kWCh + __shfl_sync(0xffffffffu, k0 + lastk, src);
        }
      }
      if (kWrite) {  // striped stores: row r = entries 32 r .. 32 r + 31 of the chunk
        const unsigned* words = reinterpret_cast<const unsigned*>(tb + ch * 32);
        int rb0 = 0, rb1 = 0;  // same-side entries in the chunk's earlier rows
#pragma unroll
        for (int r = 0; r < 8; ++r) {
          const int e = r * 32 + lane;
          const int rowlen = min(32, clen - r * 32);
          if (rowlen <= 0) break;
          const unsigned rvm = rowlen >= 32 ? 0xffffffffu : ((1u << rowlen) - 1u);
          const unsigned w = __ldg(words + r) & rvm;
          if (e < clen) {
            const bool hi = (w >> lane) & 1u;
            const int rank = hi ? rb0 + __popc(w & ltm) : rb1 + __popc(~w & rvm & ltm);
            const long long d = hi ? dbase0 + ccnt[0] + rank : dbase1 + ccnt[1] + rank;
#ifdef GBDT_FUSEDW_DEBUG
            {
              const int cc = c0 + (hi ? 0 : 1);
              const long long lo_ = (long long)a * stride_n + S.offn[cc], hi_ = lo_ + (S.offn[cc + 1] - S.offn[cc]);
              if (d < lo_ || d >= hi_)
                printf("BAD t=%d ch=%d r=%d lane=%d hi=%d rank=%d ccnt=%d,%d rb=%d,%d w=%08x clen=%d cont=%d j0=%d off=%d q0=%d len=%d\n",
                       t, ch, r, lane, (int)hi, rank, ccnt[0], ccnt[1], rb0, rb1, w, clen, (int)cont, j0, S.off[j0], q0, len);
            }
#endif
            __stcs(A.val_out + d, SG.val[e]);
            __stcs(A.ins_out + d, SG.ins[e]);
            __stcs(A.g_out + d, SG.g[e]);
          }
          rb0 += __popc(w);
          rb1 += __popc(~w & rvm);
        }
      }
      ccnt[0] += th;
      ccnt[1] += tl;
      __syncwarp();
      issue(ch + 2);  // stage st is drained
    }
    // the tile's bests -> the global records (only if they can still win)
    if (lane < 2) {
      const int q = lane;
      if (bkey[q] && bkey[q] >= __ldcg(A.gkey + c0 + q)) {
        Rec rc;
        rc.gain = eq2_gain(bGL[q], bHL[q], Gc[q], Hc[q], lam, Pc[q]);
        rc.GL = bGL[q]; rc.HL = bHL[q]; rc.cntL = bcnt[q]; rc.pos = bpos[q]; rc.value = bval[q];
        rc.attr = A.a_base + a; rc.dir = 0; rc.node = c0 + q; rc.epoch = (int)ep; rc.shard = A.shard;
        A.rec[atomicAdd(A.nrec, 1)] = rc;
        atomicMax(A.gkey + c0 + q, bkey[q]);
      }
    }
  }
}

// ============================================================================ plan + mark
// One thread: the level's segment offsets, child offsets / parents, tile count.
__global__ void k_fused_plan(FusedPlan* P, NodeTab cur, NodeTab nxt, const int32_t* __restrict__ cidx,
                             const int* __restrict__ epoch, int m, unsigned long long* lent, int lvl,
                             int* __restrict__ mcount) {
  if (threadIdx.x != 0) return;
  *mcount = 0;
  const int K = *cur.K, Kn = *nxt.K;
  P->K = K;
  P->Kn = Kn;
  int o = 0;
  for (int j = 0; j < K; ++j) {
    P->off[j] = o;
    o += cur.cnt[j];
    P->cidx[j] = cidx[j];
    if (cidx[j] >= 0) { P->pj[cidx[j]] = j; P->pj[cidx[j] + 1] = j; }
  }
  P->off[K] = o;
  int on = 0;
  for (int c = 0; c < Kn; ++c) {
    P->offn[c] = on;
    on += nxt.cnt[c];
  }
  P->offn[Kn] = on;
  P->n_act = o;
  P->stride = (o + 3) & ~3ll;
  P->n_next = on;
  P->stride_next = (on + 3) & ~3ll;
  P->tpa = (o + kFTile - 1) / kFTile;
  P->T = Kn > 0 ? m * P->tpa : 0;
  P->epoch = *epoch;
  if (lent) lent[lvl + 1] += (unsigned long long)on * (unsigned long long)m;
}

// Instance -> non-default-side bits of the splits found by k_fused (level l+1), marked from the
// parent level l's lists: child c's entries are the entries of its parent's segment on c's side
// (high child: even c), in order; the high part of c's split is those at positions <= pos.
__global__ void k_mark_fused(const FusedPlan* __restrict__ P, const int32_t* __restrict__ Kp,
                             const int32_t* __restrict__ cidx_now, const Rec* __restrict__ winner, int shard,
                             int a_base, const int32_t* __restrict__ ins, const uint32_t* __restrict__ hbit,
                             uint32_t* __restrict__ bits) {
  const int c = blockIdx.y;
  if (c >= *Kp || cidx_now[c] < 0) return;
  const Rec& w = winner[c];
  if (w.shard != shard) return;
  const int jp = P->pj[c];
  const unsigned want = (c & 1) == 0 ? 1u : 0u;
  const long long s0 = (long long)(w.attr - a_base) * P->stride + P->off[jp];
  const long long n = P->off[jp + 1] - P->off[jp];
  for (long long q = (long long)blockIdx.x * blockDim.x + threadIdx.x; q < n; q += (long long)gridDim.x * blockDim.x) {
    const long long p = s0 + q;
    const int i = ins[p];
    if (((hbit[i >> 5] >> (i & 31)) & 1u) != want) continue;
    const int high = p <= w.pos;
    if (high != w.dir) atomicOr(bits + (i >> 5), 1u << (i & 31));
  }
}

unsigned g_fused_grid[2][2] = {{0, 0}, {0, 0}};
unsigned g_agg_grid = 0;
unsigned g_fusedw_grid = 0;

template <int HM, bool W>
void set_fusedw(int sms) {
  const size_t smem = sizeof(WSmem);
  GBDT_CUDA(cudaFuncSetAttribute(k_fusedw<HM, W>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  GBDT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_fusedw<HM, W>, kWW * 32, smem));
  if (occ < 1) fail(GBDT_E_CUDA, "k_fusedw does not fit on an SM");
  const unsigned g = (unsigned)(occ * sms);
  g_fusedw_grid = g_fusedw_grid ? std::min(g_fusedw_grid, g) : g;
}

template <int HM, bool W>
void set_fused(int sms) {
  const size_t smem = sizeof(FusedSmem);
  GBDT_CUDA(cudaFuncSetAttribute(k_fused<HM, W>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  GBDT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_fused<HM, W>, kFT, smem));
  if (occ < 1) fail(GBDT_E_CUDA, "k_fused does not fit on an SM");
  g_fused_grid[HM][W ? 1 : 0] = (unsigned)std::min(occ * sms, kFusedMaxCTAs);
}

}  // namespace

size_t fused_tile_bytes(int64_t max_tiles) {
  const int64_t groups = (max_tiles + kTSGroup - 1) / kTSGroup + 1;
  return (size_t)max_tiles * (2 * sizeof(TRec) + 2 + kFT + 4) + (size_t)groups * (2 * sizeof(TRec) + 1) + 8192 +
         sizeof(Rec) * 2 * kFusedMaxK * (size_t)kFusedMaxCTAs;
}
int64_t fused_tiles(int64_t n, int m) { return (int64_t)m * ((n + kFTile - 1) / kFTile); }

void fused_carve(FusedArgs& A, void* base, int64_t max_tiles) {
  const int64_t groups = (max_tiles + kTSGroup - 1) / kTSGroup + 1;
  char* p = static_cast<char*>(base);
  auto take = [&](size_t b) { char* r = p; p += (b + 255) & ~size_t(255); return r; };
  A.cta_rec = reinterpret_cast<Rec*>(take(sizeof(Rec) * 2 * kFusedMaxK * (size_t)kFusedMaxCTAs));
  A.mcount = reinterpret_cast<int*>(take(16));
  A.mlist = reinterpret_cast<int*>(take(4 * (size_t)max_tiles));
  A.tagg = reinterpret_cast<TRec*>(take(sizeof(TRec) * max_tiles));
  A.tinc = reinterpret_cast<TRec*>(take(sizeof(TRec) * max_tiles));
  A.tgagg = reinterpret_cast<TRec*>(take(sizeof(TRec) * groups));
  A.tgcarry = reinterpret_cast<TRec*>(take(sizeof(TRec) * groups));
  A.treset = reinterpret_cast<unsigned char*>(take(max_tiles));
  A.tseen = reinterpret_cast<unsigned char*>(take(max_tiles));
  A.tgf = reinterpret_cast<unsigned char*>(take(groups));
  A.tbits = reinterpret_cast<unsigned char*>(take((size_t)kFT * max_tiles));
}

void fused_init(int sms) {
  set_fused<kHConst2, true>(sms);
  set_fused<kHConst2, false>(sms);
  set_fused<kHFromG, true>(sms);
  set_fused<kHFromG, false>(sms);
  set_fusedw<kHConst2, true>(sms);
  set_fusedw<kHConst2, false>(sms);
  set_fusedw<kHFromG, true>(sms);
  set_fusedw<kHFromG, false>(sms);
  int occ = 0;
  GBDT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_tile_agg<kHFromG>, kFT, 0));
  g_agg_grid = (unsigned)(std::max(occ, 1) * sms);
}

unsigned fused_grid(int hmode) { return std::max(g_fused_grid[hmode][0], g_fused_grid[hmode][1]); }

void fused_plan(FusedPlan* P, const NodeTab& cur, const NodeTab& nxt, const int32_t* cidx, const int* epoch, int m,
                unsigned long long* lent, int lvl, int* mcount, cudaStream_t st) {
  k_fused_plan<<<1, 32, 0, st>>>(P, cur, nxt, cidx, epoch, m, lent, lvl, mcount);
  GBDT_LAUNCH_CHECK();
  count_launch();
}

void fused_pass(const FusedArgs& A, int hmode, bool write, int64_t max_tiles, cudaStream_t st) {
  // tile sides + aggregates, the exact tile scan, then the fused pass itself
  const unsigned ga = (unsigned)std::max<int64_t>(1, std::min<int64_t>(max_tiles, g_agg_grid));
  if (hmode == kHConst2) k_tile_agg<kHConst2><<<ga, kFT, 0, st>>>(A);
  else k_tile_agg<kHFromG><<<ga, kFT, 0, st>>>(A);
  const unsigned gs = (unsigned)std::max<int64_t>(1, (max_tiles + kTSGroup - 1) / kTSGroup);
  k_tscan1<<<gs, kTSGroup, 0, st>>>(A);
  k_tscan2<<<1, kTSGroup, 0, st>>>(A);
  k_tscan3<<<gs, kTSGroup, 0, st>>>(A);
  const size_t smemw = sizeof(WSmem);
  const unsigned gw = g_fusedw_grid;
  if (!A.warp_tiles) {
  } else if (hmode == kHConst2) {
    if (write) k_fusedw<kHConst2, true><<<gw, kWW * 32, smemw, st>>>(A);
    else k_fusedw<kHConst2, false><<<gw, kWW * 32, smemw, st>>>(A);
  } else {
    if (write) k_fusedw<kHFromG, true><<<gw, kWW * 32, smemw, st>>>(A);
    else k_fusedw<kHFromG, false><<<gw, kWW * 32, smemw, st>>>(A);
  }
  const size_t smem = sizeof(FusedSmem);
  const unsigned grid = g_fused_grid[hmode][write ? 1 : 0];
  if (hmode == kHConst2) {
    if (write) k_fused<kHConst2, true><<<grid, kFT, smem, st>>>(A);
    else k_fused<kHConst2, false><<<grid, kFT, smem, st>>>(A);
  } else {
    if (write) k_fused<kHFromG, true><<<grid, kFT, smem, st>>>(A);
    else k_fused<kHFromG, false><<<grid, kFT, smem, st>>>(A);
  }
  GBDT_LAUNCH_CHECK();
  count_launch(6);
}

void fused_mark(const FusedPlan* P, const int32_t* Kp, const int32_t* cidx, const Rec* winner, int shard, int a_base,
                const int32_t* ins, const uint32_t* hbit, uint32_t* bits, int64_t n, int Kl, int sms, cudaStream_t st) {
  dim3 grid((unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256 * (int64_t)Kl), (int64_t)sms * 4)),
            (unsigned)Kl);
  k_mark_fused<<<grid, 256, 0, st>>>(P, Kp, cidx, winner, shard, a_base, ins, hbit, bits);
  GBDT_LAUNCH_CHECK();
  count_launch();
}

}  // namespace gbdt
