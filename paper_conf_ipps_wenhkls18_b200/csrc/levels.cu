// levels.cu -- the per-level streaming kernels of the hot path on sm_100a:
//
//   a3-a6 split find: segmented prefix sum of (g, h, count) over every (node,
//         attribute) segment of the level's attribute-sorted lists (Fig. 1), Eq. 2 gain at the end
//         of every run of equal values, both missing directions,
//         best split per node
//   a8    partition: order-preserving stable partition of every segment into its two
//         children; entries of new leaves are dropped
//
// Work decomposition.  An attribute list is cut into 256-entry CHUNKS (one warp: 32 lanes x 8
// consecutive entries) and 2048-entry TILES (8 chunks); neither straddles attributes.  Every
// streaming kernel is warp-granular -- a warp owns a chunk end to end and never waits for
// another warp -- so latency is hidden by warp parallelism alone:
//   k_chunk_agg   per chunk: g (h) of its entries -- gathered from the L2-resident per-instance
//                 array at the root (the only random access of the level), read from the g-list
//                 the partition carried along below it -- and the chunk's segmented aggregate
//   k_scan1/2/3   exact segmented exclusive scan of the chunk aggregates (three parallel phases)
//   k_sf          persistent tile loop over a 3-stage shared-memory ring fed by TMA 1-D bulk
//                 copies (cp.async.bulk / UBLKCP, mbarrier completion, L2 evict-first) of the
//                 tile's value list and g-list; each warp scans its chunk from its carry, ranks
//                 its run ends (Eq. 2), and posts its best candidates to a per-CTA node table
//   k_part_count / k_scan1/2/3 / k_part_plan / k_part_scatter   count -> scan -> stable scatter,
//                 the entry's g (h) moving with it
//
// Determinism.  Inside a chunk every sum has a fixed association.  Across chunks, each chunk's
// fp64 aggregate is converted ONCE to an exact 128-bit fixed-point integer (trunc(x * 2^F), F per
// tree so that every sum stays below 2^125) and carries are integer sums: exact and associative,
// so every prefix, gain and tree is bit-identical whatever the schedule, the scan decomposition or
// the attribute sharding (chunks are attribute-aligned).  Partition offsets are integer counts.
#include <algorithm>
#include <climits>

#include "kernels.cuh"

namespace gbdt {
namespace {

constexpr int kStages = 3;
constexpr int kSegCache = 32;     // segment starts/counts of a tile's attribute cached per stage
constexpr int kTabCache = 64;     // attribute tables cached in smem when m <= kTabCache
constexpr int kChunksPerTile = kTile / kChunk;  // 8 == kWarps
constexpr int kScanGroup = 1024;  // elements per CTA in the 3-phase scans
static_assert(kChunksPerTile == kWarps, "one warp per chunk of a tile");

// ============================================================================ scan algebra
struct SVf {
  double g, h;
  int c, f;  // f: contains a segment head
};
__device__ __forceinline__ SVf svf_zero() { return SVf{0.0, 0.0, 0, 0}; }
// segmented combine: a head in the right operand discards the left one
__device__ __forceinline__ SVf comb(const SVf& l, const SVf& r) {
  if (r.f) return r;
  return SVf{l.g + r.g, l.h + r.h, l.c + r.c, l.f};
}
__device__ __forceinline__ SVf shfl_up(const SVf& x, int o) {
  return SVf{__shfl_up_sync(0xffffffffu, x.g, o), __shfl_up_sync(0xffffffffu, x.h, o),
             __shfl_up_sync(0xffffffffu, x.c, o), __shfl_up_sync(0xffffffffu, x.f, o)};
}

__device__ __forceinline__ __int128 shfl_up128(__int128 v, int o) {
  const unsigned long long lo = __shfl_up_sync(0xffffffffu, (unsigned long long)v, o);
  const unsigned long long hi = __shfl_up_sync(0xffffffffu, (unsigned long long)((unsigned __int128)v >> 64), o);
  return (__int128)(((unsigned __int128)hi << 64) | lo);
}
__device__ __forceinline__ __int128 shfl_idx128(__int128 v, int l) {
  const unsigned long long lo = __shfl_sync(0xffffffffu, (unsigned long long)v, l);
  const unsigned long long hi = __shfl_sync(0xffffffffu, (unsigned long long)((unsigned __int128)v >> 64), l);
  return (__int128)(((unsigned __int128)hi << 64) | lo);
}

// Element of the exact scans: fixed-point (g, h), count, head-inside flag.  In global memory:
// 5 words  g.lo g.hi h.lo h.hi  count | f << 32 | reset-before << 33.
struct FXV {
  __int128 g, h;
  int c, f;
};
__device__ __forceinline__ FXV fxv_comb(const FXV& l, const FXV& r) {
  if (r.f) return r;
  return FXV{l.g + r.g, l.h + r.h, l.c + r.c, l.f};
}
__device__ __forceinline__ void fxv_store(unsigned long long* dst, const FXV& x, int reset) {
  dst[0] = (unsigned long long)x.g;
  dst[1] = (unsigned long long)((unsigned __int128)x.g >> 64);
  dst[2] = (unsigned long long)x.h;
  dst[3] = (unsigned long long)((unsigned __int128)x.h >> 64);
  dst[4] = (unsigned long long)(unsigned)x.c | ((unsigned long long)(x.f & 1) << 32) |
           ((unsigned long long)(reset & 1) << 33);
}
__device__ __forceinline__ FXV fxv_load(const unsigned long long* src, int* reset = nullptr) {
  const unsigned long long w = src[4];
  if (reset) *reset = (int)((w >> 33) & 1);
  return FXV{(__int128)(((unsigned __int128)src[1] << 64) | src[0]),
             (__int128)(((unsigned __int128)src[3] << 64) | src[2]), (int)(unsigned)w, (int)((w >> 32) & 1)};
}

// Carry record of a chunk as the split kernels read it: the exclusive segmented prefix converted
// to fp64 once (k_scan3), and the entry count.
struct CarryD {
  double g, h;
  int c;
};
__device__ __forceinline__ void carry_store(unsigned long long* dst5, long long i, const FXV& x, int Fg, int Fh) {
  unsigned long long* d = dst5 + 5 * i;
  d[0] = (unsigned long long)__double_as_longlong(from_fx(x.g, Fg));
  d[2] = (unsigned long long)__double_as_longlong(from_fx(x.h, Fh));
  d[4] = (unsigned long long)(unsigned)x.c | ((unsigned long long)(x.f & 1) << 32);
}
__device__ __forceinline__ CarryD carry_load(const unsigned long long* src5) {
  return CarryD{__longlong_as_double((long long)src5[0]), __longlong_as_double((long long)src5[2]),
                (int)(unsigned)src5[4]};
}

// 1/x for x > 0 (normal): hardware seed + two Newton steps (~1 ulp).  Used only to RANK the
// candidates of a chunk; the winner's Eq. 2 gain is then recomputed with IEEE divisions.
__device__ __forceinline__ double rcp_nr(double x) {
  double r;
  asm("rcp.approx.ftz.f64 %0, %1;" : "=d"(r) : "d"(x));
  double e = __fma_rn(-x, r, 1.0);
  r = __fma_rn(r, e, r);
  e = __fma_rn(-x, r, 1.0);
  return __fma_rn(r, e, r);
}

// ============================================================================ plumbing
struct TabCache {
  int use;
  int chunk_start[kTabCache + 1];
  long long col_start[kTabCache + 1];
  long long col_len[kTabCache];
};

__device__ __forceinline__ void tab_load(TabCache& tc, const TileArgs& A) {
  const bool use = A.m <= kTabCache;
  if (threadIdx.x == 0) tc.use = use;
  if (use) {
    for (int i = threadIdx.x; i <= A.m; i += blockDim.x) {
      tc.chunk_start[i] = A.tb.chunk_start[i];
      tc.col_start[i] = A.tb.col_start[i];
      if (i < A.m) tc.col_len[i] = A.tb.col_len[i];
    }
  }
}

// largest a with start[a] <= x
__device__ __forceinline__ int find_attr(const int* start, int m, int x) {
  int lo = 0, hi = m - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (start[mid] <= x) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// The chunk set of the chunk kernels: every chunk, or (short path, levels.cu k_short_*) the list of
// the chunks of the other attributes
__device__ __forceinline__ int nchunks(const Tables& tb) { return tb.lc ? *tb.nlc : *tb.C; }
__device__ __forceinline__ int chunk_at(const Tables& tb, int i) { return tb.lc ? tb.lc[i] : i; }

// Range of one chunk (all lanes compute it; the tables are in smem when m is small).
struct ChunkMeta {
  long long p0, p1, sb;
  int a, reset, more;  // more: the attribute continues after the chunk
};
__device__ __forceinline__ ChunkMeta chunk_meta(const TabCache& tc, const TileArgs& A, int K, int c) {
  const bool u = tc.use;
  const int* cs = u ? tc.chunk_start : A.tb.chunk_start;
  const int a = A.tb.chunk_attr[c];
  const long long c0 = u ? tc.col_start[a] : A.tb.col_start[a];
  const long long cl = u ? tc.col_len[a] : A.tb.col_len[a];
  const int k = c - cs[a];
  ChunkMeta M;
  M.a = a;
  M.reset = (k == 0);
  M.p0 = c0 + (long long)k * kChunk;
  M.p1 = min(M.p0 + (long long)kChunk, c0 + cl);
  M.more = M.p1 < c0 + cl;
  M.sb = (long long)a * K;
  return M;
}

// L2 prefetch of a chunk's list bytes [p0, p0 + 256) * elem (lanes take one 128-byte line each)
__device__ __forceinline__ void prefetch_chunk(const void* list, long long p0, int elem, int lane) {
  const char* b = reinterpret_cast<const char*>(list) + p0 * elem;
  // evict-last: the prefetched lines must survive the streaming traffic until the warp reads them
  // (C3 scatter 11.38 -> 11.22 ms/tree against a plain prefetch; 12.03 without prefetch)
  if (lane * 128 < kChunk * elem) asm volatile("prefetch.global.L2::evict_last [%0];" ::"l"(b + lane * 128));
}

// Segment (node) of each of the thread's items; head / piece-end / run-end masks.  ss/sc are the
// attribute's segment starts/counts; p1 bounds the piece (chunk end).
template <bool kNeedVal>
__device__ __forceinline__ void assign_segments(const long long* ss, const long long* sc, long long p1, int K,
                                                long long base, unsigned vm, const float* v, float vnext,
                                                int* sj, unsigned& hm, unsigned& pem, unsigned& rem,
                                                long long* first = nullptr) {
  hm = pem = rem = 0;
  if (!vm) return;
  int lo = 0, hi = K - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (ss[mid] <= base) lo = mid; else hi = mid - 1;
  }
  int j = lo;
  long long s0 = ss[j], se = s0 + sc[j];
  if (first) { first[0] = s0; first[1] = se; }  // segment of the thread's first entry
#pragma unroll
  for (int k = 0; k < kItems; ++k) {
    const long long p = base + k;
    if (!((vm >> k) & 1)) { sj[k] = j; continue; }
    while (p >= se) { ++j; s0 = ss[j]; se = s0 + sc[j]; }
    sj[k] = j;
    if (p == s0) hm |= 1u << k;
    const bool seg_last = (p + 1 == se);
    if (seg_last || p + 1 == p1) pem |= 1u << k;
    if (kNeedVal) {
      const float nv = (k < kItems - 1) ? v[k + 1] : vnext;
      if (seg_last || nv != v[k]) rem |= 1u << k;
    } else if (seg_last) {
      rem |= 1u << k;
    }
  }
}

// Segment holding list position p0 (the largest j with ss[j] <= p0, as the binary searches find
// it) and that segment's start/end, warp-cooperatively: with K <= 32 one coalesced load of the
// attribute's segment table and a ballot instead of log2(K) dependent loads.  Warp-uniform result.
struct SegOf {
  int j;
  long long s0, se;
};
__device__ __forceinline__ SegOf warp_seg(const long long* ss, const long long* sc, int K, long long p0, int lane) {
  SegOf r;
  if (K <= 32) {
    const long long s = lane < K ? ss[lane] : LLONG_MAX;
    const long long c = lane < K ? sc[lane] : 0;
    const unsigned msk = __ballot_sync(0xffffffffu, s <= p0);
    r.j = 31 - __clz(msk | 1u);
    r.s0 = __shfl_sync(0xffffffffu, s, r.j);
    r.se = r.s0 + __shfl_sync(0xffffffffu, c, r.j);
  } else {
    int lo = 0, hi = K - 1;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (ss[mid] <= p0) lo = mid; else hi = mid - 1;
    }
    r.j = lo;
    r.s0 = ss[lo];
    r.se = r.s0 + sc[lo];
  }
  return r;
}

// ============================================================================ a4: chunk aggregates
#ifndef GBDT_AGG_SHORT
#define GBDT_AGG_SHORT 1
#endif
// Short chunk (<= 32 entries, K <= 32: the typical sparse list): lane i holds entry
// p0 + i, the segment structure comes from the attribute's segment table held one segment per
// lane (as in sf_short), and the segmented sums run over the lanes instead of the 8-items-per-lane
// layout, whose loops and scans a 20-entry list pays in full.  Same outputs as the general path:
// descriptor, exact chunk aggregate, g-list at the root, present totals of the ending segments.
template <int HMODE, bool kGather>
__device__ __forceinline__ void agg_short(const SplitArgs& A, const ChunkMeta& M, int c, int K, int lane, int Fg,
                                          int Fh, unsigned long long pol_keep, float vnx) {
  const long long p0 = M.p0;
  const int len = (int)(M.p1 - p0);
  const bool valid = lane < len;
  const long long p = p0 + lane;
  double g = 0.0, h = 0.0;
  if (valid) {
    if (kGather) {
      const int id = __ldcs(A.t.ins + p);
      g = ld_keep(A.g + id, pol_keep);
      h = HMODE == kHGather ? ld_keep(A.h + id, pol_keep) : hess_of<HMODE>(g);
      __stcs(A.glist + p, g);
      if (HMODE == kHGather) __stcs(A.hlist + p, h);
    } else {
      g = __ldcs(A.glist + p);
      h = HMODE == kHGather ? __ldcs(A.hlist + p) : hess_of<HMODE>(g);
    }
  }
  const long long* ss = (const long long*)(A.t.tb.seg_start + M.sb);
  const long long* sc = (const long long*)(A.t.tb.seg_cnt + M.sb);
  const long long s_l = lane < K ? ss[lane] : LLONG_MAX;
  const long long c_l = lane < K ? sc[lane] : 0;
  // segment of the chunk's first entry: the largest j with ss[j] <= p0 (warp_seg's choice)
  const unsigned le0 = __ballot_sync(0xffffffffu, s_l <= p0);
  const int j0 = 31 - __clz(le0 | 1u);
  const long long s0 = __shfl_sync(0xffffffffu, s_l, j0);
  const long long se0 = s0 + __shfl_sync(0xffffffffu, c_l, j0);
  const int head0 = s0 == p0 ? 1 : 0;
  if (M.p1 <= se0) {  // one segment: the aggregate is the whole chunk
    double lg = g, lh = h;
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      lg = lg + __shfl_xor_sync(0xffffffffu, lg, o);
      lh = lh + __shfl_xor_sync(0xffffffffu, lh, o);
    }
    if (lane == 0) {
      ChunkDesc d;
      d.p0 = p0;
      d.se = se0;
      d.len = len;
      d.a = M.a;
      d.jf = j0 | (head0 ? kDescHead0 : 0) | kDescSingle | (M.more ? kDescNext : 0);
      d.vnext = vnx;
      A.desc[c] = d;
      fxv_store(A.cagg + 5ll * c, FXV{to_fx(lg, Fg), to_fx(lh, Fh), len, head0}, M.reset);
      if (A.segEnd && M.p1 == se0) {
        const long long s = M.sb + j0;
        A.segPG_out[s] = lg;
        A.segPH_out[s] = lh;
        A.segEnd[s] = head0 ? -1 : c;
      }
    }
    return;
  }
  if (lane == 0) {  // the chunk crosses a segment boundary: k_sf_gen's
    ChunkDesc d;
    d.p0 = p0;
    d.se = se0;
    d.len = len;
    d.a = M.a;
    d.jf = j0 | (head0 ? kDescHead0 : 0) | (M.more ? kDescNext : 0);
    d.vnext = vnx;
    A.desc[c] = d;
    A.genlist[atomicAdd(A.ngen, 1)] = c;
  }
  // heads inside the chunk (first entries of non-empty segments) and the lane's segment piece
  const bool starts = lane < K && c_l > 0 && s_l >= p0 && s_l < p0 + len;
  const unsigned hm = __reduce_or_sync(0xffffffffu, starts ? (1u << (int)(s_l - p0)) : 0u);
  const unsigned upto = hm & (0xffffffffu >> (31 - lane));
  const int hpos = upto ? 31 - __clz(upto) : -1;  // last head at or before the lane
  const int sl = hpos >= 0 ? hpos : 0;
  double ig = g, ih = h;
  int icn = valid ? 1 : 0;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const double yg = __shfl_up_sync(0xffffffffu, ig, o), yh = __shfl_up_sync(0xffffffffu, ih, o);
    const int yc = __shfl_up_sync(0xffffffffu, icn, o);
    if (lane - o >= sl) { ig = yg + ig; ih = yh + ih; icn += yc; }
  }
  // lanes past the end hold zeros in the last piece: lane 31 has the aggregate since the last head
  if (lane == 31) fxv_store(A.cagg + 5ll * c, FXV{to_fx(ig, Fg), to_fx(ih, Fh), icn, hm != 0u}, M.reset);
  if (A.segEnd) {
    // the lane's segment: the owner of the head at hpos (unique: heads are non-empty segments)
    int j = j0;
    unsigned o = __ballot_sync(0xffffffffu, starts);
    while (o) {
      const int l = __ffs(o) - 1;
      o &= o - 1;
      const long long sll = __shfl_sync(0xffffffffu, s_l, l);
      if (hpos >= 0 && sll - p0 == hpos) j = l;
    }
    const long long se = __shfl_sync(0xffffffffu, s_l, j & 31) + __shfl_sync(0xffffffffu, c_l, j & 31);
    if (valid && p + 1 == se) {  // present totals of the segments ending here (see k_seg_totals)
      const long long s = M.sb + j;
      A.segPG_out[s] = ig;
      A.segPH_out[s] = ih;
      A.segEnd[s] = hpos >= 0 ? -1 : c;
    }
  }
}

// One warp per chunk: g (h) of its entries -- gathered at the root (L2 evict-last) and laid out as
// the chunk's g-list, read from the partition-carried g-list below -- and the chunk's segmented
// aggregate (sum since its last segment head, fixed association) as an exact fixed-point value.
template <int HMODE, bool kGather>
#ifndef GBDT_AGG_CTAS
#define GBDT_AGG_CTAS 4  // list-reading instantiation (missing values, below the root): <= 64 registers
#endif                   // (~96 B of spills), C4a chunk pass 2.01 -> 1.78 ms/tree; the root gather stays at
                         // 3 CTAs/SM (C3 root 3.33 vs 3.37 ms/tree at 4)
__global__ void __launch_bounds__(kThreads, kGather ? 3 : GBDT_AGG_CTAS) k_chunk_agg(SplitArgs A) {
  __shared__ TabCache tc;
  const int lane = threadIdx.x & 31;
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0 || C == 0) return;
  const int Fg = A.fx[0], Fh = A.fx[1];
  const unsigned long long pol_keep = policy_evict_last();
  tab_load(tc, A.t);
  __syncthreads();
  const int nw = (gridDim.x * blockDim.x) >> 5;
  const int NC = nchunks(A.t.tb);
  for (int i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < NC; i += nw) {
    const int c = chunk_at(A.t.tb, i);
    const ChunkMeta M = chunk_meta(tc, A.t, K, c);
    const long long p1 = M.p1;
    const long long base = M.p0 + (long long)lane * kItems;
    if (!kGather && i + nw < NC) {  // the warp's next chunk streams into L2 meanwhile
      const ChunkMeta Mn = chunk_meta(tc, A.t, K, chunk_at(A.t.tb, i + nw));
      prefetch_chunk(A.glist, Mn.p0, 8, lane);
      if (HMODE == kHGather) prefetch_chunk(A.hlist, Mn.p0, 8, lane);
    }
    // value after the chunk (same attribute), for the descriptor; loaded early
    const float vnx = (lane == 0 && M.more && !A.rle) ? __ldg(A.t.val + p1) : 0.f;
#if GBDT_AGG_SHORT
    if (p1 - M.p0 <= 32 && K <= 32) {
      agg_short<HMODE, kGather>(A, M, c, K, lane, Fg, Fh, pol_keep, vnx);
      continue;
    }
#endif
    unsigned vm = 0;
    double g[kItems], h[kItems];
#pragma unroll
    for (int k = 0; k < kItems; ++k) { g[k] = 0.0; h[k] = 0.0; }
    if (base < p1) {
      if (kGather) {
        const int4 i0 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base));
        const int4 i1 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base + 4));
        const int id[kItems] = {i0.x, i0.y, i0.z, i0.w, i1.x, i1.y, i1.z, i1.w};
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
          if (base + k < p1) {
            vm |= 1u << k;
            g[k] = ld_keep(A.g + id[k], pol_keep);
            h[k] = HMODE == kHGather ? ld_keep(A.h + id[k], pol_keep) : hess_of<HMODE>(g[k]);
          }
        }
        if (base + kItems <= p1) {  // lists are padded to 4 entries only: never write past the chunk
          double2* go = reinterpret_cast<double2*>(A.glist + base);
#pragma unroll
          for (int q = 0; q < kItems / 2; ++q) __stcs(go + q, make_double2(g[2 * q], g[2 * q + 1]));
          if (HMODE == kHGather) {
            double2* ho = reinterpret_cast<double2*>(A.hlist + base);
#pragma unroll
            for (int q = 0; q < kItems / 2; ++q) __stcs(ho + q, make_double2(h[2 * q], h[2 * q + 1]));
          }
        } else {
#pragma unroll
          for (int k = 0; k < kItems; ++k)
            if (base + k < p1) {
              A.glist[base + k] = g[k];
              if (HMODE == kHGather) A.hlist[base + k] = h[k];
            }
        }
      } else {
        // every list is padded to 4 entries: the lane's two 4-entry halves are loaded whole
        const double2* gi = reinterpret_cast<const double2*>(A.glist + base);
        const double2* hi2 = reinterpret_cast<const double2*>(A.hlist + base);
        const bool two = base + 4 < p1;
#pragma unroll
        for (int q = 0; q < kItems / 2; ++q) {
          if (q < 2 || two) {
            const double2 x = __ldcs(gi + q);
            g[2 * q] = x.x; g[2 * q + 1] = x.y;
            if (HMODE == kHGather) { const double2 y = __ldcs(hi2 + q); h[2 * q] = y.x; h[2 * q + 1] = y.y; }
          }
        }
        const int nv = (int)min((long long)kItems, p1 - base);
        vm = (1u << nv) - 1u;
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
          if (HMODE != kHGather) h[k] = hess_of<HMODE>(g[k]);
          if (k >= nv) { g[k] = 0.0; h[k] = 0.0; }
        }
      }
    }
    // segment of the chunk's first entry (warp-uniform search; the attribute's table is in L1)
    const long long* ss = (const long long*)(A.t.tb.seg_start + M.sb);
    const long long* sc = (const long long*)(A.t.tb.seg_cnt + M.sb);
    const SegOf sg = warp_seg(ss, sc, K, M.p0, lane);
    const int j0 = sg.j;
    const long long s0 = sg.s0, se = sg.se;
    const int len = (int)(p1 - M.p0);
    if (p1 <= se) {
      // one segment: the aggregate is the whole chunk (a head can only be its first entry)
      double lg = 0.0, lh = 0.0;
#pragma unroll
      for (int k = 0; k < kItems; ++k) { lg = lg + g[k]; lh = lh + h[k]; }  // invalid items are 0
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        lg = lg + __shfl_xor_sync(0xffffffffu, lg, o);
        lh = lh + __shfl_xor_sync(0xffffffffu, lh, o);
      }
      if (lane == 0) {
        ChunkDesc d;
        d.p0 = M.p0;
        d.se = se;
        d.len = len;
        d.a = M.a;
        d.jf = j0 | (s0 == M.p0 ? kDescHead0 : 0) | kDescSingle | (M.more ? kDescNext : 0);
        d.vnext = vnx;
        A.desc[c] = d;
        fxv_store(A.cagg + 5ll * c, FXV{to_fx(lg, Fg), to_fx(lh, Fh), len, s0 == M.p0 ? 1 : 0}, M.reset);
        // with missing values k_sf_gen takes every chunk but k_sf_short's: list them all
        if (A.segEnd) A.genlist[atomicAdd(A.ngen, 1)] = c;
        if (A.segEnd && p1 == se) {  // the segment ends here: its present totals (see k_seg_totals)
          const long long s = M.sb + j0;
          A.segPG_out[s] = lg;
          A.segPH_out[s] = lh;
          A.segEnd[s] = s0 == M.p0 ? -1 : c;
        }
      }
      continue;
    }
    int sj[kItems];
    unsigned hm, pem, rem;
    float vd[kItems];
    assign_segments<false>(ss, sc, p1, K, base, vm, vd, 0.f, sj, hm, pem, rem);
    if (lane == 0) {  // the chunk crosses a segment boundary: k_sf_gen's
      ChunkDesc d;
      d.p0 = M.p0;
      d.se = se;
      d.len = len;
      d.a = M.a;
      d.jf = j0 | (s0 == M.p0 ? kDescHead0 : 0) | (M.more ? kDescNext : 0);
      d.vnext = vnx;
      A.desc[c] = d;
      A.genlist[atomicAdd(A.ngen, 1)] = c;
    }
    SVf run = svf_zero();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1)) continue;
      if ((hm >> k) & 1) { run.g = g[k]; run.h = h[k]; run.c = 1; run.f = 1; }
      else { run.g = run.g + g[k]; run.h = run.h + h[k]; run.c += 1; }
    }
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const SVf y = shfl_up(run, o);
      if (lane >= o) run = comb(y, run);
    }
    if (lane == 31)
      fxv_store(A.cagg + 5ll * c, FXV{to_fx(run.g, Fg), to_fx(run.h, Fh), run.c, run.f}, M.reset);
    if (A.segEnd) {
      // present totals of the segments ending in this chunk: the in-chunk segmented sum at their
      // last entry; k_seg_totals adds the carry when the segment began in an earlier chunk
      SVf exc = shfl_up(run, 1);
      if (lane == 0) exc = svf_zero();
      SVf loc = svf_zero();
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (!((vm >> k) & 1)) continue;
        if ((hm >> k) & 1) { loc.g = g[k]; loc.h = h[k]; loc.c = 1; loc.f = 1; }
        else { loc.g = loc.g + g[k]; loc.h = loc.h + h[k]; loc.c += 1; }
        if ((rem >> k) & 1) {
          const long long s = M.sb + sj[k];
          A.segPG_out[s] = loc.f ? loc.g : exc.g + loc.g;
          A.segPH_out[s] = loc.f ? loc.h : exc.h + loc.h;
          A.segEnd[s] = (loc.f || exc.f) ? -1 : c;
        }
      }
    }
  }
}

// ============================================================================ exact scans
// Segmented exclusive scan over chunk elements x_c with head-inside flags f_c and reset-before
// flags r_c (first chunk of an attribute):
//   I_c = (f_c | r_c) ? x_c : I_{c-1} + x_c,    E_c = r_c ? 0 : I_{c-1}.
// Integer arithmetic, so the result does not depend on how the scan is decomposed:
//   k_scan1: per group of kScanGroup elements, the group's segmented aggregate
//   k_scan2: one warp, exclusive segmented scan over the group aggregates (in place)
//   k_scan3: per group, every element's exclusive value from the group's carry
struct PK {  // packed count element (partition): hi | lo << 32
  unsigned long long v;
  int f;
};

template <bool kFx>
struct ScanOps;
template <>
struct ScanOps<true> {
  using T = FXV;
  static constexpr int W = 5;
  static __device__ T zero() { return FXV{0, 0, 0, 0}; }
  static __device__ T load(const unsigned long long* a, long long i, int& r) {
    T x = fxv_load(a + W * i, &r);
    x.f |= r;
    return x;
  }
  static __device__ T load_plain(const unsigned long long* a, long long i) { return fxv_load(a + W * i); }
  static __device__ void store(unsigned long long* a, long long i, const T& x) { fxv_store(a + W * i, x, 0); }
  static __device__ T comb(const T& l, const T& r) { return fxv_comb(l, r); }
  static __device__ T up(const T& x, int o) {
    return FXV{shfl_up128(x.g, o), shfl_up128(x.h, o), __shfl_up_sync(0xffffffffu, x.c, o),
               __shfl_up_sync(0xffffffffu, x.f, o)};
  }
  static __device__ T idx(const T& x, int l) {
    return FXV{shfl_idx128(x.g, l), shfl_idx128(x.h, l), __shfl_sync(0xffffffffu, x.c, l),
               __shfl_sync(0xffffffffu, x.f, l)};
  }
};
template <>
struct ScanOps<false> {
  using T = PK;
  static constexpr int W = 2;
  static __device__ T zero() { return PK{0ull, 0}; }
  static __device__ T load(const unsigned long long* a, long long i, int& r) {
    r = (int)(a[W * i + 1] & 1);
    return PK{a[W * i], r};
  }
  static __device__ T load_plain(const unsigned long long* a, long long i) {
    return PK{a[W * i], (int)(a[W * i + 1] & 1)};
  }
  static __device__ void store(unsigned long long* a, long long i, const T& x) {
    a[W * i] = x.v;
    a[W * i + 1] = (unsigned long long)x.f;
  }
  static __device__ T comb(const T& l, const T& r) { return r.f ? r : PK{l.v + r.v, l.f}; }
  static __device__ T up(const T& x, int o) {
    return PK{__shfl_up_sync(0xffffffffu, x.v, o), __shfl_up_sync(0xffffffffu, x.f, o)};
  }
  static __device__ T idx(const T& x, int l) {
    return PK{__shfl_sync(0xffffffffu, x.v, l), __shfl_sync(0xffffffffu, x.f, l)};
  }
};

template <bool kFx>
__global__ void __launch_bounds__(kThreads) k_scan1(const int32_t* __restrict__ Cp, const unsigned long long* __restrict__ in,
                                                   unsigned long long* __restrict__ gagg) {
  using O = ScanOps<kFx>;
  using T = typename O::T;
  constexpr int kPer = kScanGroup / kThreads;
  __shared__ T wt[kWarps];
  const int C = *Cp, lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const long long g0 = (long long)blockIdx.x * kScanGroup;
  if (g0 >= C) return;
  T run = O::zero();
  for (int k = 0; k < kPer; ++k) {
    const long long i = g0 + (long long)threadIdx.x * kPer + k;
    if (i < C) { int r; run = O::comb(run, O::load(in, i, r)); }
  }
  for (int o = 1; o < 32; o <<= 1) {
    const T y = O::up(run, o);
    if (lane >= o) run = O::comb(y, run);
  }
  if (lane == 31) wt[wid] = run;
  __syncthreads();
  if (threadIdx.x == 0) {
    T acc = O::zero();
    for (int w = 0; w < kWarps; ++w) acc = O::comb(acc, wt[w]);
    O::store(gagg, blockIdx.x, acc);
  }
}

// One block of kScan2Threads: every thread takes a contiguous run of group aggregates, so the
// dependent chain is ceil(G / kScan2Threads) elements plus two warp scans (not G / 32 warp scans).
constexpr int kScan2Threads = 1024;
template <bool kFx>
__global__ void __launch_bounds__(kScan2Threads) k_scan2(const int32_t* __restrict__ Cp, unsigned long long* __restrict__ gagg) {
  using O = ScanOps<kFx>;
  using T = typename O::T;
  __shared__ T wt[kScan2Threads / 32];
  const int C = *Cp;
  const int G = (C + kScanGroup - 1) / kScanGroup;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int per = (G + kScan2Threads - 1) / kScan2Threads;
  const int i0 = threadIdx.x * per, i1 = min(G, i0 + per);
  T run = O::zero();
  for (int i = i0; i < i1; ++i) run = O::comb(run, O::load_plain(gagg, i));
  T inc = run;
  for (int o = 1; o < 32; o <<= 1) {
    const T y = O::up(inc, o);
    if (lane >= o) inc = O::comb(y, inc);
  }
  T ex = O::up(inc, 1);
  if (lane == 0) ex = O::zero();
  if (lane == 31) wt[wid] = inc;
  __syncthreads();
  if (wid == 0) {  // exclusive scan of the warp totals
    const T x = wt[lane];
    T wi = x;
    for (int o = 1; o < 32; o <<= 1) {
      const T y = O::up(wi, o);
      if (lane >= o) wi = O::comb(y, wi);
    }
    T we = O::up(wi, 1);
    if (lane == 0) we = O::zero();
    __syncwarp();
    wt[lane] = we;
  }
  __syncthreads();
  T pre = O::comb(wt[wid], ex);  // everything before the thread's first element
  for (int i = i0; i < i1; ++i) {
    const T x = O::load_plain(gagg, i);
    O::store(gagg, i, pre);
    pre = O::comb(pre, x);
  }
}
// kFx: the carries are written as fp64 values (word 0: g, word 2: h, word 4: count | flags),
// converted once here from the exact fixed-point prefix instead of in every consumer
template <bool kFx>
__global__ void __launch_bounds__(kThreads) k_scan3(const int32_t* __restrict__ Cp, const unsigned long long* __restrict__ in,
                                                   const unsigned long long* __restrict__ gcar,
                                                   unsigned long long* __restrict__ out, const int32_t* __restrict__ fx) {
  using O = ScanOps<kFx>;
  using T = typename O::T;
  constexpr int kPer = kScanGroup / kThreads;
  __shared__ T wt[kWarps];
  __shared__ T wc[kWarps];
  const int C = *Cp, lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const long long g0 = (long long)blockIdx.x * kScanGroup;
  if (g0 >= C) return;
  T x[kPer];
  int r[kPer];
  T run = O::zero();
#pragma unroll
  for (int k = 0; k < kPer; ++k) {
    const long long i = g0 + (long long)threadIdx.x * kPer + k;
    r[k] = 0;
    x[k] = O::zero();
    if (i < C) x[k] = O::load(in, i, r[k]);
    run = O::comb(run, x[k]);
  }
  T inc = run;
  for (int o = 1; o < 32; o <<= 1) {
    const T y = O::up(inc, o);
    if (lane >= o) inc = O::comb(y, inc);
  }
  T ex = O::up(inc, 1);
  if (lane == 0) ex = O::zero();
  if (lane == 31) wt[wid] = inc;
  __syncthreads();
  if (threadIdx.x == 0) {
    T acc = O::load_plain(gcar, blockIdx.x);
    for (int w = 0; w < kWarps; ++w) { wc[w] = acc; acc = O::comb(acc, wt[w]); }
  }
  __syncthreads();
  T prev = O::comb(wc[wid], ex);  // inclusive value before this thread's first element
#pragma unroll
  for (int k = 0; k < kPer; ++k) {
    const long long i = g0 + (long long)threadIdx.x * kPer + k;
    if (i < C) {
      if constexpr (kFx) carry_store(out, i, r[k] ? O::zero() : prev, fx[0], fx[1]);
      else O::store(out, i, r[k] ? O::zero() : prev);
    }
    prev = O::comb(prev, x[k]);
  }
}

// ============================================================================ a3-a6: split find
// Two kernels per level (both warp-granular: a warp owns one 256-entry chunk at a time and never
// waits for another warp):
//   k_sf_fast  every chunk that lies inside ONE segment (nearly all chunks of dense data): the
//              chunk's value list and g-list stream through a per-warp 2-stage shared-memory ring
//              fed by TMA 1-D bulk copies (UBLKCP + mbarrier, L2 evict-first); plain warp scans,
//              candidates ranked by a Newton-reciprocal score, exact Eq. 2 for the chunk's winner
//   k_sf_gen   every other chunk (chunks that cross segment boundaries; all chunks when values are
//              missing, where both default directions need the segments' present totals):
//              segmented scans and a log-time per-segment argmax, direct vector loads
// Node bests are merged per CTA in shared memory (a per-node lock; posts are rare: one per chunk
// and segment) and flushed once per CTA.
constexpr int kWarpK = 32;  // CTA node tables when K <= kWarpK (d <= 6); else global records

struct NodeBest {
  double G[kWarpK], H[kWarpK], P[kWarpK];
  int C[kWarpK];
};

struct NodeV {
  double G, H, P;
  int C;
};
__device__ __forceinline__ NodeV node_v(const NodeBest& B, const SplitArgs& A, int K, int j) {
  if (K <= kWarpK) return NodeV{B.G[j], B.H[j], B.P[j], B.C[j]};
  return NodeV{A.nodes.G[j], A.nodes.H[j], A.nodes.pterm[j], A.nodes.cnt[j]};
}

__device__ __forceinline__ void nb_init(NodeBest& B, const SplitArgs& A, int K) {
  for (int j = threadIdx.x; j < kWarpK; j += blockDim.x) {
    if (j < K) { B.G[j] = A.nodes.G[j]; B.H[j] = A.nodes.H[j]; B.P[j] = A.nodes.pterm[j]; B.C[j] = A.nodes.cnt[j]; }
  }
}

__device__ __forceinline__ bool rec_better(unsigned long long gk, const Rec& r, unsigned long long gk0, const Rec& r0) {
  return gk > gk0 || (gk == gk0 && tie_key(r.attr, r.value, r.dir) < tie_key(r0.attr, r0.value, r0.dir));
}

// One candidate record into the global record list (K > kWarpK: too many nodes for the per-warp
// tables); k_pick_tie / k_pick_best merge them in the R12 order.
__device__ __forceinline__ void post_global(const SplitArgs& A, const Rec& r) {
  const int gs = atomicAdd(A.nrec, 1);
  A.rec[gs] = r;
  atomicMax(A.gkey + r.node, gain_key(r.gain));
}

// With K <= kWarpK every warp keeps its own best record per node (one writer: no lock, no race);
// at the end the CTA merges its warps' tables in the R12 order and posts one record per node.
__device__ __forceinline__ void merge_warp_tables(const SplitArgs& A, int K, unsigned long long (*wgk)[kWarpK],
                                                  Rec (*wrec)[kWarpK]) {
  __syncthreads();
  for (int j = threadIdx.x; j < K; j += blockDim.x) {
    int bw = -1;
    for (int w = 0; w < kWarps; ++w)
      if (wgk[w][j] && (bw < 0 || rec_better(wgk[w][j], wrec[w][j], wgk[bw][j], wrec[bw][j]))) bw = w;
    if (bw >= 0) {
      const int gs = atomicAdd(A.nrec, 1);
      A.rec[gs] = wrec[bw][j];
      atomicMax(A.gkey + j, wgk[bw][j]);
    }
  }
}

// rank score of a split: GL^2/(HL+l) + GR^2/(HR+l) = 2 Eq. 2 + G^2/(H+l); one Newton reciprocal
__device__ __forceinline__ double split_score(double GL, double HL, double G, double H, double lam) {
  const double dl = HL + lam, dr = (H - HL) + lam, GR = G - GL;
  return __dmul_rn(__fma_rn(GL * GL, dr, __dmul_rn(GR * GR, dl)), rcp_nr(__dmul_rn(dl, dr)));
}

// value of list position p from the level's runs (RLE): the run holding it, searched between
// the runs holding the first entries of chunk cg and of the next chunk
__device__ __forceinline__ void rle_values(const Tables& tb, int cg, long long p0, long long len, bool has_next,
                                           long long base, int K, int sb_end_seg, float* v, float& vnext) {
  int lo = tb.run_chunk[cg];
  int hi = has_next ? tb.run_chunk[cg + 1] : tb.seg_run[sb_end_seg] - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (tb.run_pos[mid] <= base) lo = mid; else hi = mid - 1;
  }
  int r = lo;
  long long rend = tb.run_pos[r] + tb.run_len[r];
  float rv = tb.run_val[r];
  const long long pend = p0 + len + (has_next ? 1 : 0);
#pragma unroll
  for (int k = 0; k <= kItems; ++k) {
    const long long p = base + k;
    if (p >= pend) { if (k < kItems) v[k] = 0.f; continue; }
    while (p >= rend) { ++r; rend = tb.run_pos[r] + tb.run_len[r]; rv = tb.run_val[r]; }
    if (k < kItems) v[k] = rv; else vnext = rv;
  }
}

// A lane's 8 consecutive entries [8 lane, 8 lane + 8) of a chunk staged in shared memory, read
// as 16-byte pieces in natural order.  The 64-byte lane stride makes these 4-way (g) and 2-way (v)
// bank conflicts; a lane-rotated order avoids them but needs ~40 selects per chunk to rotate back,
// and the kernel is issue bound: natural order measured 6.41 vs 6.66 ms/tree of split on C3.
__device__ __forceinline__ void lds_blocked8(const double* chunk, int lane, double* out) {
  const double2* p = reinterpret_cast<const double2*>(chunk) + lane * 4;
#pragma unroll
  for (int j = 0; j < 4; ++j) {
    const double2 z = p[j];
    out[2 * j] = z.x;
    out[2 * j + 1] = z.y;
  }
}
__device__ __forceinline__ void lds_blocked8f(const float* chunk, int lane, float* out) {
  const float4* p = reinterpret_cast<const float4*>(chunk) + lane * 2;
  const float4 a0 = p[0], a1 = p[1];
  out[0] = a0.x; out[1] = a0.y; out[2] = a0.z; out[3] = a0.w;
  out[4] = a1.x; out[5] = a1.y; out[6] = a1.z; out[7] = a1.w;
}

// ---------------------------------------------------------------------------- k_sf_fast
constexpr int kFS = 2;  // stages per warp
template <bool kH>
struct __align__(16) FastWarp {
  float val[kFS][kChunk + 4];  // + the value after the chunk
  double g[kFS][kChunk];
  double h[kH ? kFS : 1][kH ? kChunk : 2];
  unsigned long long carry[kFS][6];
  ChunkDesc d[4];
  unsigned long long bar[kFS];
  unsigned rend[kChunk / 32];  // RLE: bit p - p0 set iff entry p is the last entry of its run
};
template <bool kH>
struct FastSmem {
  FastWarp<kH> w[kWarps];
  NodeBest B;
  unsigned long long wgk[kWarps][kWarpK];  // per-warp node bests (K <= kWarpK)
  Rec wrec[kWarps][kWarpK];
};

template <int HMODE, bool kRLE>
__global__ void __launch_bounds__(kThreads, 3) k_sf_fast(SplitArgs A) {
  constexpr bool kH = HMODE == kHGather;
  extern __shared__ __align__(128) unsigned char smem_raw[];
  FastSmem<kH>& S = *reinterpret_cast<FastSmem<kH>*>(smem_raw);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0 || C == 0) return;
  const int epoch = *A.epochp;
  const int Fg = A.fx[0], Fh = A.fx[1];
  const double lam = A.lam;
  FastWarp<kH>& W = S.w[wid];
  nb_init(S.B, A, K);
  for (int j = threadIdx.x; j < kWarps * kWarpK; j += blockDim.x) S.wgk[j / kWarpK][j % kWarpK] = 0ull;
  if (lane == 0) {
    for (int s = 0; s < kFS; ++s) mbar_init(&W.bar[s], 1);
    fence_mbar_init();
  }
  __syncthreads();
  const int NW = gridDim.x * kWarps;
  const int gw = blockIdx.x * kWarps + wid;
  const unsigned long long pol = policy_evict_first();
  auto chunk = [&](int i) { return gw + i * NW; };
  // descriptor (and carry) prefetch into the warp's rings
  auto fetch = [&](int i, bool with_desc, bool with_carry) {
    const int c = chunk(i);
    if (c < C) {
      if (with_desc && lane < 4) cp_async8(reinterpret_cast<unsigned long long*>(&W.d[i & 3]) + lane,
                                          reinterpret_cast<const unsigned long long*>(A.desc + c) + lane, pol);
      if (with_carry && lane < 5) cp_async8(&W.carry[i & 1][lane], A.carry + 5ll * c + lane, pol);
    }
  };
  // TMA of chunk i's lists into stage i & 1 (single-segment chunks only)
  auto issue = [&](int i) {
    const int c = chunk(i);
    if (lane == 0 && c < C) {
      const ChunkDesc& d = W.d[i & 3];
      if (d.jf & kDescSingle) {
        const int st = i & 1;
        const uint32_t n = (uint32_t)((d.len + 3) & ~3);
        fence_proxy_async();
        mbar_arrive_expect_tx(&W.bar[st], (kRLE ? 0u : 4u * n) + 8u * n + (kH ? 8u * n : 0u));
        if (!kRLE) tma_load_1d(W.val[st], A.t.val + d.p0, 4u * n, &W.bar[st], pol);
        tma_load_1d(W.g[st], A.glist + d.p0, 8u * n, &W.bar[st], pol);
        if (kH) tma_load_1d(W.h[st], A.hlist + d.p0, 8u * n, &W.bar[st], pol);
      }
    }
  };
  fetch(0, true, true);
  fetch(1, true, true);
  fetch(2, true, false);
  cp_async_commit();
  cp_async_wait<0>();
  __syncwarp();
  issue(0);
  issue(1);
  uint32_t ph = 0;
  for (int i = 0; chunk(i) < C; ++i) {
    const int st = i & 1;
    const ChunkDesc& d = W.d[i & 3];
    const int jf = d.jf;
    if (jf & kDescSingle) {
      mbar_wait(&W.bar[st], (ph >> st) & 1);
      ph ^= 1u << st;
      const long long p0 = d.p0, se = d.se;
      const int len = d.len;
      const int j = jf & 0xffff;
      float* sv = W.val[st];
      const int q0 = lane * kItems;
      double g[kItems], hk[kItems];
      float v[kItems], vn = 0.f;
      if (!kRLE && lane == 0) sv[len] = d.vnext;  // the value after the chunk follows its last entry
      __syncwarp();
      lds_blocked8(W.g[st], lane, g);
      if (kH) lds_blocked8(W.h[st], lane, hk);
      unsigned rmask = 0;  // RLE: the lane's items that end a run (the runs are the candidates)
      int rb = 0, re = 0;
      if (kRLE) {
        // the runs touching the chunk (one per lane, usually one or two in all): each marks its
        // last entry, so no value is decompressed per entry
        const int cg = chunk(i);
        rb = A.t.tb.run_chunk[cg];
        re = (jf & kDescNext) ? A.t.tb.run_chunk[cg + 1] : A.t.tb.seg_run[d.a * K + K] - 1;
        if (lane < kChunk / 32) W.rend[lane] = 0u;
        __syncwarp();
        for (int r = rb + lane; r <= re; r += 32) {
          const long long e = A.t.tb.run_pos[r] + A.t.tb.run_len[r] - 1 - p0;
          if (e >= 0 && e < len) atomicOr(&W.rend[e >> 5], 1u << (e & 31));
        }
        __syncwarp();
        rmask = (W.rend[lane >> 2] >> ((lane & 3) * 8)) & 0xffu;
#pragma unroll
        for (int k = 0; k < kItems; ++k) v[k] = 0.f;
      } else {
        lds_blocked8f(sv, lane, v);
        vn = __shfl_down_sync(0xffffffffu, v[0], 1);
        if (lane == 31) vn = sv[kChunk];
      }
      if (!kH) {
#pragma unroll
        for (int k = 0; k < kItems; ++k) hk[k] = hess_of<HMODE>(g[k]);
      }
      if (q0 + kItems > len) {  // the chunk's tail: items past its end contribute nothing
#pragma unroll
        for (int k = 0; k < kItems; ++k)
          if (q0 + k >= len) { g[k] = 0.0; hk[k] = 0.0; }
      }
      // pass 1: the lane's sums (fixed tree association), warp scan -> the lane's exclusive prefix
      double wg = ((g[0] + g[1]) + (g[2] + g[3])) + ((g[4] + g[5]) + (g[6] + g[7]));
      double wh = ((hk[0] + hk[1]) + (hk[2] + hk[3])) + ((hk[4] + hk[5]) + (hk[6] + hk[7]));
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const double yg = __shfl_up_sync(0xffffffffu, wg, o), yh = __shfl_up_sync(0xffffffffu, wh, o);
        if (lane >= o) { wg = yg + wg; wh = yh + wh; }
      }
      double eg = __shfl_up_sync(0xffffffffu, wg, 1), eh = __shfl_up_sync(0xffffffffu, wh, 1);
      if (lane == 0) { eg = 0.0; eh = 0.0; }
      const bool head0 = (jf & kDescHead0) != 0;
      double bg, bh;
      int bc;
      {
        const CarryD cx = carry_load(W.carry[st]);
        bg = (head0 ? 0.0 : cx.g) + eg;
        bh = (head0 ? 0.0 : cx.h) + eh;
        bc = (head0 ? 0 : cx.c) + min(q0, len);  // entries of the segment before the lane's first item
      }
      const NodeV nv = node_v(S.B, A, K, j);
      // Candidates are run ends (the next value differs) with a non-empty low side: there are no
      // missing values on this path, so that excludes exactly the segment's last entry.
      const int nc = min(((p0 + len == se) ? len - 1 : len) - q0, nv.C - 1 - bc);
      // pass 2: prefix at every item, candidates ranked inside the lane by the score num/den
      // compared by cross-multiplication (no division), num = GL^2 (HR+l) + GR^2 (HL+l),
      // den = (HL+l)(HR+l); only the winning item index is carried
      const double Hl = nv.H + lam;
      unsigned cm = 0;  // the lane's candidates: run ends with a non-empty low side
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        const float nx = k < kItems - 1 ? v[k + 1] : vn;
        if (k < nc && (kRLE ? ((rmask >> k) & 1u) != 0u : nx != v[k])) cm |= 1u << k;
      }
      double pg = bg, phh = bh, bnum = -1.0, bden = 1.0;
      int bk = -1;
      double wb = -INFINITY;
      int wq = INT_MAX;
      // Low-cardinality lists (long runs of equal values, RLE-shaped data) have chunks without any
      // run end: the whole warp skips the scoring (only run ends are candidates).
      if (__any_sync(0xffffffffu, cm != 0u)) {
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
          pg = pg + g[k];
          phh = phh + hk[k];
          const double dl = phh + lam, dr = Hl - phh, GR = nv.G - pg;
          const double num = __fma_rn(__dmul_rn(pg, pg), dr, __dmul_rn(__dmul_rn(GR, GR), dl)), den = __dmul_rn(dl, dr);
          if (((cm >> k) & 1u) && __dmul_rn(num, bden) > __dmul_rn(bnum, den)) { bnum = num; bden = den; bk = k; }
        }
        wb = bk < 0 ? -INFINITY : __dmul_rn(bnum, rcp_nr(bden));
        wq = bk < 0 ? INT_MAX : q0 + bk;
        // warp argmax (largest score, then smallest position) by three integer reductions on the
        // order-preserving bit pattern of the score (scores are >= +0 or -inf, never NaN)
        unsigned long long kb = (unsigned long long)__double_as_longlong(wb);
        kb = (kb >> 63) ? ~kb : (kb | 0x8000000000000000ull);
        const unsigned mhi = __reduce_max_sync(0xffffffffu, (unsigned)(kb >> 32));
        const unsigned mlo = __reduce_max_sync(0xffffffffu, (unsigned)(kb >> 32) == mhi ? (unsigned)kb : 0u);
        const bool top = (unsigned)(kb >> 32) == mhi && (unsigned)kb == mlo;
        wq = (int)__reduce_min_sync(0xffffffffu, top ? (unsigned)wq : 0xffffffffu);
        unsigned long long km = ((unsigned long long)mhi << 32) | mlo;
        km = (km >> 63) ? (km & 0x7fffffffffffffffull) : ~km;
        wb = __longlong_as_double((long long)km);
      }
      // Can the chunk's best still beat node j's best so far in this CTA?  Its approximate gain
      // (the ranking score, ~1e-15 relative) must come within a 1e-12 relative slack of it;
      // otherwise the exact Eq. 2 evaluation and the post are skipped (warp-uniform test).
      bool promising = wq != INT_MAX;
      if (promising && K <= kWarpK) {
        const unsigned long long cur = S.wgk[wid][j];  // this warp's best so far (written by it only)
        if (cur) {
          const double ga = 0.5 * (wb - nv.P), slack = 1e-12 * (fabs(wb) + fabs(nv.P));
          promising = ga + slack >= key_gain(cur);
        }
      }
      if (promising && bk >= 0 && wq == q0 + bk) {
        // the winner's prefix, by the same sequence of additions as pass 2
        double xg = bg, xh = bh;
        float xv = 0.f;
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
          if (k <= bk) { xg = xg + g[k]; xh = xh + hk[k]; }
          if (!kRLE && k == bk) xv = v[k];
        }
        if (kRLE) {  // the winner ends a run of this chunk: that run's value
          const long long pw = p0 + q0 + bk;
          for (int r2 = rb; r2 <= re; ++r2)
            if (A.t.tb.run_pos[r2] + A.t.tb.run_len[r2] - 1 == pw) { xv = A.t.tb.run_val[r2]; break; }
        }
        Rec r;
        r.GL = xg;
        r.HL = xh;
        r.cntL = bc + bk + 1;
        r.gain = eq2_gain(xg, xh, nv.G, nv.H, lam, nv.P);
        r.value = xv;
        r.attr = A.t.a_base + d.a;
        r.dir = 0;
        r.node = j;
        r.epoch = epoch;
        r.shard = A.shard;
        r.pos = p0 + bk + q0;
        if (K <= kWarpK) {
          const unsigned long long gk = gain_key(r.gain);
          if (rec_better(gk, r, S.wgk[wid][j], S.wrec[wid][j])) { S.wgk[wid][j] = gk; S.wrec[wid][j] = r; }
        } else {
          post_global(A, r);
        }
      }
    }
    __syncwarp();  // stage st and descriptor slot i & 3 are free
    cp_async_wait<0>();  // descriptor of chunk i + 2 (and carry of chunk i + 1)
    __syncwarp();
    issue(i + 2);
    fetch(i + 3, true, false);
    fetch(i + 2, false, true);
    cp_async_commit();
  }
  cp_async_wait<0>();
  if (K <= kWarpK) merge_warp_tables(A, K, S.wgk, S.wrec);
}

// ---------------------------------------------------------------------------- short chunks
// A chunk of at most 32 entries (the typical list of a sparse attribute, "many small
// segments") with K <= 32 nodes: lane i holds entry p0 + i.  Segment heads come from the
// attribute's segment table (lane l holds segment l), the segmented scan and the per-segment
// argmax run over the lanes, so the work is ~1/8 of the 8-items-per-lane general path.
template <int HMODE, bool kMissing, bool kRLE>
__device__ __forceinline__ void sf_short(const SplitArgs& A, NodeBest& B, unsigned long long* wgk, Rec* wrec, int c,
                                         const ChunkDesc& d, int K, int lane, int epoch, int Fg, int Fh, double lam) {
  constexpr bool kH = HMODE == kHGather;
  const long long p0 = d.p0;
  const int len = d.len;
  const long long sb = (long long)d.a * K;
  const long long* ss = (const long long*)(A.t.tb.seg_start + sb);
  const long long* sc = (const long long*)(A.t.tb.seg_cnt + sb);
  const bool valid = lane < len;
  const long long p = p0 + lane;
  // the attribute's segment table: lane l holds segment l
  const long long s_l = lane < K ? ss[lane] : LLONG_MAX;
  const long long c_l = lane < K ? sc[lane] : 0;
  double lPG = 0.0, lPH = 0.0;
  if (kMissing && lane < K) { lPG = A.segPG[sb + lane]; lPH = A.segPH[sb + lane]; }
  // head mask: the first entries of the non-empty segments that start inside the chunk
  const bool starts = lane < K && c_l > 0 && s_l >= p0 && s_l < p0 + len;
  unsigned hbit = starts ? (1u << (int)(s_l - p0)) : 0u;
  const unsigned hm = __reduce_or_sync(0xffffffffu, hbit);
  // segment of the chunk's first entry (largest j with ss[j] <= p0) and of every lane
  const unsigned le0 = __ballot_sync(0xffffffffu, s_l <= p0);
  const int j0 = 31 - __clz(le0 | 1u);
  // lane -> segment: the head at or before the lane (its segment is the lane l that owns it)
  const unsigned upto = hm & (0xffffffffu >> (31 - lane));
  const int hpos = upto ? 31 - __clz(upto) : -1;  // position of the last head <= lane
  // the segment starting at chunk position q is the largest l with s_l == p0 + q and c_l > 0
  const unsigned own = __ballot_sync(0xffffffffu, starts);
  int j = j0;
  {
    // find l with starts && s_l - p0 == hpos: scan the owners (at most K <= 32)
    unsigned o = own;
    while (o) {
      const int l = __ffs(o) - 1;
      o &= o - 1;
      const long long sl = __shfl_sync(0xffffffffu, s_l, l);
      if (hpos >= 0 && sl - p0 == hpos) j = l;
    }
  }
  const long long sj0 = __shfl_sync(0xffffffffu, s_l, j & 31), cj0 = __shfl_sync(0xffffffffu, c_l, j & 31);
  const long long se = sj0 + cj0;  // end of the lane's segment
  const double PG = kMissing ? __shfl_sync(0xffffffffu, lPG, j & 31) : 0.0;
  const double PH = kMissing ? __shfl_sync(0xffffffffu, lPH, j & 31) : 0.0;
  // values, g, h
  float v = 0.f;
  double g = 0.0, h = 0.0;
  if (valid) {
    if (kRLE) {
      int lo = A.t.tb.run_chunk[c];
      int hi = (d.jf & kDescNext) ? A.t.tb.run_chunk[c + 1] : A.t.tb.seg_run[sb + K] - 1;
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (A.t.tb.run_pos[mid] <= p) lo = mid; else hi = mid - 1;
      }
      v = A.t.tb.run_val[lo];
    } else {
      v = __ldcs(A.t.val + p);
    }
    g = __ldcs(A.glist + p);
    h = kH ? __ldcs(A.hlist + p) : hess_of<HMODE>(g);
  }
  float vn = __shfl_down_sync(0xffffffffu, v, 1);
  if (lane == len - 1) {
    if (d.jf & kDescNext) {
      if (kRLE) {
        const int rc = A.t.tb.run_chunk[c + 1];
        vn = A.t.tb.run_val[rc];
      } else {
        vn = d.vnext;
      }
    } else {
      vn = v;  // no entry after the chunk: the segment ends here (seg_last below)
    }
  }
  // segmented inclusive scan over the lanes; lanes before the first head continue the carry
  const int sl = hpos >= 0 ? hpos : 0;  // first lane of the lane's segment piece
  double ig = g, ih = h;
  int icn = valid ? 1 : 0;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const double yg = __shfl_up_sync(0xffffffffu, ig, o), yh = __shfl_up_sync(0xffffffffu, ih, o);
    const int yc = __shfl_up_sync(0xffffffffu, icn, o);
    if (lane - o >= sl) { ig = yg + ig; ih = yh + ih; icn += yc; }
  }
  if (hpos < 0) {
    const CarryD cx = carry_load(A.carry + 5ll * c);
    ig = cx.g + ig;
    ih = cx.h + ih;
    icn = cx.c + icn;
  }
  // candidate: the end of a run of equal values (or of the segment), both directions when the
  // segment has missing values
  const bool seg_last = valid && (p + 1 == se);
  const bool cand = valid && (seg_last || vn != v);
  const NodeV nv = node_v(B, A, K, j);
  double best = -INFINITY;
  int bd = 0;
  bool ok = false;
  if (cand) {
    if (icn >= 1 && nv.C - icn >= 1) { best = split_score(ig, ih, nv.G, nv.H, lam); ok = true; }
    if (kMissing) {
      const int cM = nv.C - (int)cj0;
      const int cL1 = icn + cM;
      if (cM > 0 && cL1 >= 1 && nv.C - cL1 >= 1) {
        const double g1 = split_score(ig + (nv.G - PG), ih + (nv.H - PH), nv.G, nv.H, lam);
        if (!ok || g1 > best) { best = g1; bd = 1; ok = true; }
      }
    }
  }
  // per-segment argmax: segmented max-scan of (score, lane); earlier lane = larger value (R12)
  double lg = ok ? best : -INFINITY;
  int lq = ok ? lane : INT_MAX;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const double yg = __shfl_up_sync(0xffffffffu, lg, o);
    const int yq = __shfl_up_sync(0xffffffffu, lq, o);
    if (lane - o >= sl && (yg > lg || (yg == lg && yq < lq))) { lg = yg; lq = yq; }
  }
  // the last lane of each segment piece posts its winner
  const bool piece_end = valid && (lane == len - 1 || ((hm >> (lane + 1)) & 1u) || seg_last);
  const int q = piece_end && lq != INT_MAX ? lq : lane;
  const double wg = __shfl_sync(0xffffffffu, ig, q), wh = __shfl_sync(0xffffffffu, ih, q);
  const int wc = __shfl_sync(0xffffffffu, icn, q), wd = __shfl_sync(0xffffffffu, bd, q);
  const float wv = __shfl_sync(0xffffffffu, v, q);
  if (piece_end && lq != INT_MAX) {
    Rec r;
    r.value = wv;
    r.attr = A.t.a_base + d.a;
    r.dir = wd;
    r.node = j;
    r.epoch = epoch;
    r.shard = A.shard;
    r.pos = p0 + lq;
    if (wd) {
      r.GL = wg + (nv.G - PG);
      r.HL = wh + (nv.H - PH);
      r.cntL = wc + (nv.C - (int)cj0);
    } else {
      r.GL = wg; r.HL = wh; r.cntL = wc;
    }
    r.gain = eq2_gain(r.GL, r.HL, nv.G, nv.H, lam, nv.P);
    const unsigned long long gk = gain_key(r.gain);
    if (rec_better(gk, r, wgk[j], wrec[j])) { wgk[j] = gk; wrec[j] = r; }
  }
  __syncwarp();
}

// ---------------------------------------------------------------------------- k_sf_short
// The short chunks of k_sf_gen's chunk set in a kernel of their own.  In the general kernel the
// ~6 k-instruction body stalled on instruction fetch ("no_instructions") a third of the time on
// C4a, whose ~1.35 M lists per level are nearly all short, at 2 CTAs per SM (128 registers); here
// the loop runs from sf_short's small footprint at the occupancy its registers allow.
#ifndef GBDT_SF_SHORT_KERNEL
#define GBDT_SF_SHORT_KERNEL 1
#endif
template <int HMODE, bool kMissing, bool kRLE>
#ifndef GBDT_SFSHORT_CTAS
#define GBDT_SFSHORT_CTAS 0  // 0: the compiler's choice (a minimum of 1 CTA/SM would let it take more registers)
#endif
#if GBDT_SFSHORT_CTAS > 0
#define LB_GBDT_SFSHORT_CTAS __launch_bounds__(kThreads, GBDT_SFSHORT_CTAS)
#else
#define LB_GBDT_SFSHORT_CTAS __launch_bounds__(kThreads)
#endif
__global__ void LB_GBDT_SFSHORT_CTAS k_sf_short(SplitArgs A) {
  __shared__ NodeBest B;
  __shared__ unsigned long long wgk[kWarps][kWarpK];
  __shared__ Rec wrec[kWarps][kWarpK];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0 || C == 0 || K > kWarpK) return;
  const int epoch = *A.epochp;
  const int Fg = A.fx[0], Fh = A.fx[1];
  nb_init(B, A, K);
  for (int j = threadIdx.x; j < kWarps * kWarpK; j += blockDim.x) wgk[j / kWarpK][j % kWarpK] = 0ull;
  __syncthreads();
  const int nw = (gridDim.x * blockDim.x) >> 5;
  const int n = kMissing ? nchunks(A.t.tb) : *A.ngen;  // k_sf_gen's chunk set
  // 32 chunks per warp step, lane l testing chunk bt + l * nbat (strided, so the chunks of one long
  // list spread over the warps); the warp then runs the short ones
  // (only when the chunks outnumber the warps 32 to 1: a short list of heavy chunks, e.g. the
  // segment-crossing chunks of dense data, stays one chunk per warp)
  const int bw = n >= 32 * nw ? 32 : 1;
  const int nbat = (n + bw - 1) / bw;
  for (int bt = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; bt < nbat; bt += nw) {
    const int ii = bt + lane * nbat;
    int cc = 0;
    bool take = false;
    if (lane < bw && ii < n) {
      cc = kMissing ? chunk_at(A.t.tb, ii) : A.genlist[ii];
      take = A.desc[cc].len <= 32;
    }
    unsigned todo = __ballot_sync(0xffffffffu, take);
    while (todo) {
      const int c = __shfl_sync(0xffffffffu, cc, __ffs(todo) - 1);
      todo &= todo - 1;
      const ChunkDesc d = A.desc[c];
      sf_short<HMODE, kMissing, kRLE>(A, B, wgk[wid], wrec[wid], c, d, K, lane, epoch, Fg, Fh, A.lam);
    }
  }
  __syncthreads();  // merge the warp tables, one record per node and CTA
  for (int j = threadIdx.x; j < K; j += blockDim.x) {
    int bw = -1;
    for (int w = 0; w < kWarps; ++w)
      if (wgk[w][j] && (bw < 0 || rec_better(wgk[w][j], wrec[w][j], wgk[bw][j], wrec[bw][j]))) bw = w;
    if (bw >= 0) {
      const int gs = atomicAdd(A.nrec, 1);
      A.rec[gs] = wrec[bw][j];
      atomicMax(A.gkey + j, wgk[bw][j]);
    }
  }
}

// ---------------------------------------------------------------------------- short attributes
// The typical attribute of a sparse data set has a handful of entries ("many small
// segments"; C4a: 1.08 M of its 1.13 M non-empty lists hold <= 32, 0.78 M of them <= 4), so a warp
// per chunk spends ~500 instructions and several dependent table walks per list whatever its
// length.  These attributes (ShortList, fixed at the root: lists only shrink) take a path of their
// own at levels 0-5 (K <= 32): a warp takes a BATCH of 32/W attributes of similar root length (W =
// the batch's longest root list rounded up to a power of two), a group of W lanes per attribute,
// lane e on entry e of the list.  The entry's node j comes from a byte list carried with the
// entries (ShortList::jl, written by the scatter), so segment heads and ends are lane compares and
// no segment table is walked; the attribute's list start and length are the only table reads.
// The arithmetic is k_sf_short's over a chunk that is the whole list (and agg_short's for the
// present totals), in the same association, so trees are bit-identical to the chunk kernels'.
struct SLane {
  int a;        // attribute (-1: none)
  long long p;  // list position of the lane's entry
  bool valid;
  int j;        // node of the entry
  int hs, se;   // first / last lane of the entry's segment
  int lw;       // log2 W
  unsigned hm;  // segment heads of the warp
  unsigned gm;  // the lane's group
  long long p0; // list start of the lane's attribute
};
__device__ __forceinline__ SLane short_lane(const ShortList& S, const Tables& tb, int bi, int lane) {
  const int2 b = S.batch[bi];
  SLane L;
  L.lw = b.y >> 16;
  const int W = 1 << L.lw, sub = lane >> L.lw, e = lane & (W - 1);
  L.gm = W == 32 ? 0xffffffffu : ((1u << W) - 1u) << (sub * W);
  L.a = sub < (b.y & 0xffff) ? S.attrs[b.x + sub] : -1;
  long long len = 0;
  L.p0 = 0;
  if (L.a >= 0) {
    L.p0 = S.inplace ? S.cs0[L.a] : tb.col_start[L.a];
    len = S.inplace ? S.cl0[L.a] : tb.col_len[L.a];
  }
  L.valid = e < len;
  L.p = L.p0 + e;
  L.j = (L.valid && S.jl) ? (int)S.jl[L.p] : 0;
  if (S.inplace && S.jl) {
    // in-place lists: the group's lanes sorted by node, stably (= the partitioned list), the
    // entries of nodes that became leaves (0xff) and the lanes past the list at the end
    const int key = (L.valid && L.j != 0xff) ? L.j : 63;
    unsigned m = L.gm;
    int less = 0;
#pragma unroll
    for (int bt = 5; bt >= 0; --bt) {
      const unsigned bal = __ballot_sync(0xffffffffu, (key >> bt) & 1);
      if ((key >> bt) & 1) { less += __popc(m & ~bal); m &= bal; } else { m &= ~bal; }
    }
    const int dest = sub * W + less + __popc(m & ((1u << lane) - 1u));
    unsigned cand = 0xffffffffu;  // the lane whose entry lands on this lane
#pragma unroll
    for (int bt = 0; bt < 5; ++bt) {
      const unsigned bal = __ballot_sync(0xffffffffu, (dest >> bt) & 1);
      cand &= ((lane >> bt) & 1) ? bal : ~bal;
    }
    const int src = __ffs(cand) - 1;
    const int ks = __shfl_sync(0xffffffffu, key, src);
    L.valid = ks != 63;
    L.j = L.valid ? ks : 0;
    L.p = L.p0 + (src & (W - 1));
  }
  const int jp = __shfl_up_sync(0xffffffffu, L.j, 1);
  L.hm = __ballot_sync(0xffffffffu, L.valid && (e == 0 || jp != L.j));
  const unsigned vm = __ballot_sync(0xffffffffu, L.valid) & L.gm;
  const unsigned le = lane == 31 ? 0xffffffffu : (2u << lane) - 1u;  // lanes <= lane
  const unsigned hb = L.hm & le, nh = L.hm & ~le & L.gm;
  L.hs = hb ? 31 - __clz(hb) : lane;
  L.se = nh ? __ffs(nh) - 2 : (vm ? 31 - __clz(vm) : lane);
  return L;
}

template <int HMODE, bool kGather>
#ifndef GBDT_SSPLIT_CTAS
#define GBDT_SSPLIT_CTAS 4  // <= 64 registers: C4a split 4.92 -> 4.21 ms/tree
#endif
__global__ void __launch_bounds__(kThreads, GBDT_SSPLIT_CTAS) k_short_split(SplitArgs A, ShortList S) {
  constexpr bool kH = HMODE == kHGather;
  __shared__ NodeBest B;
  __shared__ unsigned long long wgk[kWarps][kWarpK];
  __shared__ Rec wrec[kWarps][kWarpK];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int K = *A.t.Kp;
  if (K == 0 || K > kWarpK || S.nb == 0) return;
  const int epoch = *A.epochp;
  const double lam = A.lam;
  nb_init(B, A, K);
  for (int j = threadIdx.x; j < kWarps * kWarpK; j += blockDim.x) wgk[j / kWarpK][j % kWarpK] = 0ull;
  __syncthreads();
  const unsigned long long pol_keep = policy_evict_last();
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int bi = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; bi < S.nb; bi += nw) {
    const SLane L = short_lane(S, A.t.tb, bi, lane);
    const int W = 1 << L.lw;
    float v = 0.f;
    double g = 0.0, h = 0.0;
    if (L.valid) {
      // in-place lists: root values and the short lists' own g-list, at root positions
      double* const gl = S.inplace ? S.gsh : A.glist;
      double* const hl = S.inplace ? S.hsh : A.hlist;
      v = __ldcs((S.inplace ? S.val0 : A.t.val) + L.p);
      if (kGather) {
        const int id = __ldcs((S.inplace ? S.ins0 : A.t.ins) + L.p);
        g = ld_keep(A.g + id, pol_keep);
        h = kH ? ld_keep(A.h + id, pol_keep) : hess_of<HMODE>(g);
        __stcs(gl + L.p, g);
        if (kH) __stcs(hl + L.p, h);
      } else {
        g = __ldcs(gl + L.p);
        h = kH ? __ldcs(hl + L.p) : hess_of<HMODE>(g);
      }
    }
    // segmented inclusive scan (k_sf_short's association)
    double ig = g, ih = h;
    for (int o = 1; o < W; o <<= 1) {
      const double yg = __shfl_up_sync(0xffffffffu, ig, o), yh = __shfl_up_sync(0xffffffffu, ih, o);
      if (lane - o >= L.hs) { ig = yg + ig; ih = yh + ih; }
    }
    const int icn = lane - L.hs + 1, cseg = L.se - L.hs + 1;
    // present totals of the segment (agg_short's association: a butterfly when the list is one
    // segment, else the scan at the segment's last entry)
    const bool one = __popc(L.hm & L.gm) == 1;
    double tg = g, th = h;
    for (int o = W >> 1; o; o >>= 1) {
      tg = tg + __shfl_xor_sync(0xffffffffu, tg, o);
      th = th + __shfl_xor_sync(0xffffffffu, th, o);
    }
    const double sg = __shfl_sync(0xffffffffu, ig, L.se), sh = __shfl_sync(0xffffffffu, ih, L.se);
    const double PG = one ? tg : sg, PH = one ? th : sh;
    const float vn = __shfl_down_sync(0xffffffffu, v, 1);
    const bool seg_last = L.valid && lane == L.se;
    const bool cand = L.valid && (seg_last || vn != v);
    const NodeV nv = node_v(B, A, K, L.j);
    double best = -INFINITY;
    int bd = 0;
    bool ok = false;
    if (cand) {
      if (icn >= 1 && nv.C - icn >= 1) { best = split_score(ig, ih, nv.G, nv.H, lam); ok = true; }
      const int cM = nv.C - cseg;
      const int cL1 = icn + cM;
      if (cM > 0 && cL1 >= 1 && nv.C - cL1 >= 1) {
        const double g1 = split_score(ig + (nv.G - PG), ih + (nv.H - PH), nv.G, nv.H, lam);
        if (!ok || g1 > best) { best = g1; bd = 1; ok = true; }
      }
    }
    // per-segment argmax, earlier lane (larger value, R12) on equal scores
    double lg = ok ? best : -INFINITY;
    int lq = ok ? lane : INT_MAX;
    for (int o = 1; o < W; o <<= 1) {
      const double yg = __shfl_up_sync(0xffffffffu, lg, o);
      const int yq = __shfl_up_sync(0xffffffffu, lq, o);
      if (lane - o >= L.hs && (yg > lg || (yg == lg && yq < lq))) { lg = yg; lq = yq; }
    }
    const bool post = seg_last && lq != INT_MAX;
    const int q = post ? lq : lane;
    const double wg = __shfl_sync(0xffffffffu, ig, q), wh = __shfl_sync(0xffffffffu, ih, q);
    const int wd = __shfl_sync(0xffffffffu, bd, q);
    const float wv = __shfl_sync(0xffffffffu, v, q);
    const long long wp = __shfl_sync(0xffffffffu, L.p, q);  // (in-place lists: lanes are sorted)
    Rec r;
    unsigned long long gk = 0ull;
    if (post) {
      const int wc = q - L.hs + 1;
      r.value = wv;
      r.attr = A.t.a_base + L.a;
      r.dir = wd;
      r.node = L.j;
      r.epoch = epoch;
      r.shard = A.shard;
      r.pos = wp;
      if (wd) {
        r.GL = wg + (nv.G - PG);
        r.HL = wh + (nv.H - PH);
        r.cntL = wc + (nv.C - cseg);
      } else {
        r.GL = wg; r.HL = wh; r.cntL = wc;
      }
      r.gain = eq2_gain(r.GL, r.HL, nv.G, nv.H, lam, nv.P);
      gk = gain_key(r.gain);
    }
    // the warp's node table, one group at a time (the segments of one list are distinct nodes)
    unsigned pm = __ballot_sync(0xffffffffu, post);
    while (pm) {
      const int g0 = (__ffs(pm) - 1) >> L.lw;
      const unsigned gmask = W == 32 ? 0xffffffffu : ((1u << W) - 1u) << (g0 * W);
      if (post && (lane >> L.lw) == g0 && rec_better(gk, r, wgk[wid][L.j], wrec[wid][L.j])) {
        wgk[wid][L.j] = gk;
        wrec[wid][L.j] = r;
      }
      pm &= ~gmask;
      __syncwarp();
    }
  }
  __syncthreads();  // merge the warp tables, one record per node and CTA
  for (int jj = threadIdx.x; jj < K; jj += blockDim.x) {
    int bw = -1;
    for (int w = 0; w < kWarps; ++w)
      if (wgk[w][jj] && (bw < 0 || rec_better(wgk[w][jj], wrec[w][jj], wgk[bw][jj], wrec[bw][jj]))) bw = w;
    if (bw >= 0) {
      const int gs = atomicAdd(A.nrec, 1);
      A.rec[gs] = wrec[bw][jj];
      atomicMax(A.gkey + jj, wgk[bw][jj]);
    }
  }
}

// In-place short lists (ShortList::inplace): the partition only moves every entry's node index to
// its child's (0xff when its node became a leaf); the lists themselves stay where they are
__global__ void __launch_bounds__(kThreads) k_short_update(PartArgs A, ShortList S) {
  const int K = *A.t.Kp;
  if (K == 0 || K > kWarpK || S.nb == 0) return;
  const int lane = threadIdx.x & 31;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int bi = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; bi < S.nb; bi += nw) {
    const int2 b = S.batch[bi];
    const int lw = b.y >> 16, W = 1 << lw, sub = lane >> lw, e = lane & (W - 1);
    if (sub >= (b.y & 0xffff)) continue;
    const int a = S.attrs[b.x + sub];
    if (e >= S.cl0[a]) continue;
    const long long p = S.cs0[a] + e;
    const int j = S.jl ? (int)S.jl[p] : 0;
    if (j == 0xff) continue;
    const uint8_t sd = __ldg(A.side + __ldcs(S.ins0 + p));
    const int c = A.cidx[j];
    S.jl_out[p] = (sd == 0 || c < 0) ? (uint8_t)0xff : (uint8_t)(sd == 1 ? c : c + 1);
  }
}

// Partition count of the short lists: per segment, its entries of each side (segH / segL of the
// plan) by ballots over the segment's lanes
__global__ void __launch_bounds__(kThreads) k_short_count(PartArgs A, ShortList S) {
  const int K = *A.t.Kp;
  if (K == 0 || K > kWarpK || S.nb == 0) return;
  const int lane = threadIdx.x & 31;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int bi = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; bi < S.nb; bi += nw) {
    const SLane L = short_lane(S, A.t.tb, bi, lane);
    const uint8_t sd = L.valid ? __ldg(A.side + __ldcs(A.t.ins + L.p)) : 0;
    const unsigned bh = __ballot_sync(0xffffffffu, sd == 1), bl = __ballot_sync(0xffffffffu, sd == 2);
    if (L.valid && lane == L.se) {
      const unsigned m = (L.se == 31 ? 0xffffffffu : (2u << L.se) - 1u) & ~((1u << L.hs) - 1u);
      const long long s = (long long)L.a * K + L.j;
      A.segH[s] = __popc(bh & m);
      A.segL[s] = __popc(bl & m);
    }
  }
}

// Stable scatter of the short lists: rank among the segment's same-side entries by
// ballot; the entries' next-level node index goes with them (ShortList::jl_out)
template <int HMODE>
__global__ void __launch_bounds__(kThreads) k_short_scatter(PartArgs A, ShortList S) {
  constexpr bool kH = HMODE == kHGather;
  const int K = *A.t.Kp;
  if (K == 0 || K > kWarpK || S.nb == 0) return;
  const int lane = threadIdx.x & 31;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int bi = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; bi < S.nb; bi += nw) {
    const SLane L = short_lane(S, A.t.tb, bi, lane);
    int id = 0;
    uint8_t sd = 0;
    if (L.valid) {
      id = __ldcs(A.t.ins + L.p);
      sd = __ldg(A.side + id);
    }
    const unsigned bh = __ballot_sync(0xffffffffu, sd == 1), bl = __ballot_sync(0xffffffffu, sd == 2);
    if (sd) {
      const bool hi = sd == 1;
      const unsigned below = ((1u << lane) - 1u) & ~((1u << L.hs) - 1u);
      const int rk = __popc((hi ? bh : bl) & below);
      const long long s = (long long)L.a * K + L.j;
      const long long d = (hi ? A.out_hi[s] : A.out_lo[s]) + rk;
      __stcs(A.val_out + d, __ldcs(A.t.val + L.p));
      __stcs(A.ins_out + d, id);
      __stcs(A.g_out + d, __ldcs(A.g_in + L.p));
      if (kH) __stcs(A.h_out + d, __ldcs(A.h_in + L.p));
      if (S.jl_out) {
        const int c = A.cidx[L.j];
        S.jl_out[d] = (uint8_t)(hi ? c : c + 1);
      }
    }
  }
}

// ---------------------------------------------------------------------------- k_sf_gen
#ifndef GBDT_GEN_CTAS
// 3 CTAs per SM (<= 85 registers; the missing-value variant does not spill): C4a split
// 5.16 -> 4.11 ms/tree (the kernel stalls on fixed-latency dependencies and instruction fetch,
// so more warps per SM pay), C4b 0.44 -> 0.47
#define GBDT_GEN_CTAS 3
#endif
#ifndef GBDT_GEN_DYN
#define GBDT_GEN_DYN 1  // dynamic claim of the chunk steps (missing values)
#endif
#ifndef GBDT_GEN_COMPACT
#define GBDT_GEN_COMPACT 1
#endif
template <int HMODE, bool kMissing, bool kTotals, bool kRLE>
__global__ void __launch_bounds__(kThreads, GBDT_GEN_CTAS) k_sf_gen(SplitArgs A) {
  constexpr bool kH = HMODE == kHGather;
  __shared__ NodeBest B;
  __shared__ unsigned char flg[kWarps][kChunk];
  // per-warp best per node: a chunk lies in one attribute, whose segments belong to distinct
  // nodes, so a warp never posts two candidates for one node at once (no atomics, no locks)
  __shared__ unsigned long long wgk[kTotals ? 1 : kWarps][kWarpK];
  __shared__ Rec wrec[kTotals ? 1 : kWarps][kWarpK];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0 || C == 0) return;
  const int epoch = *A.epochp;
  const int Fg = A.fx[0], Fh = A.fx[1];
  const double lam = A.lam;
  nb_init(B, A, K);
  if (!kTotals)
    for (int j = threadIdx.x; j < kWarps * kWarpK; j += blockDim.x) wgk[j / kWarpK][j % kWarpK] = 0ull;
  __syncthreads();
  const int nw = (gridDim.x * blockDim.x) >> 5;
  // the chunks k_chunk_agg listed: with missing values every chunk of the general layout (the
  // short ones are k_sf_short's), else those that cross segments; the totals pass takes all
  constexpr bool kAll = kTotals;
  const int n = kAll ? nchunks(A.t.tb) : *A.ngen;
  // 32 chunks per warp step (lane l tests chunk bt + l * nbat); the short ones are k_sf_short's,
  // so they cost one descriptor word here instead of a dependent descriptor load each
  // (only when the chunks outnumber the warps 32 to 1: a short list of heavy chunks, e.g. the
  // segment-crossing chunks of dense data, stays one chunk per warp)
  const int bw = n >= 32 * nw ? 32 : 1;
  const int nbat = (n + bw - 1) / bw;
  constexpr bool kDyn = GBDT_GEN_DYN && kMissing && !kTotals;
  auto claim = [&]() {
    int x = 0;
    if (lane == 0) x = atomicAdd(A.t.counter, 1);
    return __shfl_sync(0xffffffffu, x, 0);
  };
  for (int bt = kDyn ? claim() : (blockIdx.x * blockDim.x + threadIdx.x) >> 5; bt < nbat; bt = kDyn ? claim() : bt + nw) {
    const int ii = bt + lane * nbat;
    int cc = 0;
    bool take = false;
    if (lane < bw && ii < n) {
      cc = kAll ? chunk_at(A.t.tb, ii) : A.genlist[ii];
      take = kTotals || !GBDT_SF_SHORT_KERNEL || !kMissing || !(A.desc[cc].len <= 32 && K <= kWarpK);
    }
    unsigned todo = __ballot_sync(0xffffffffu, take);
    while (todo) {
    const int c = __shfl_sync(0xffffffffu, cc, __ffs(todo) - 1);
    todo &= todo - 1;
    const ChunkDesc d = A.desc[c];
    const long long p0 = d.p0;
    const long long cp1 = p0 + d.len;
    const long long sb = (long long)d.a * K;
#if GBDT_SF_SHORT_KERNEL
    if (kMissing && !kTotals && d.len <= 32 && K <= kWarpK) continue;  // k_sf_short's (sparse lists)
#else
    if (!kTotals && d.len <= 32 && K <= kWarpK) {  // short chunk (sparse lists): one entry per lane
      sf_short<HMODE, kMissing, kRLE>(A, B, wgk[wid], wrec[wid], c, d, K, lane, epoch, Fg, Fh, lam);
      continue;
    }
#endif
    const long long base = p0 + lane * kItems;
    const long long* ss = (const long long*)(A.t.tb.seg_start + sb);
    const long long* sc = (const long long*)(A.t.tb.seg_cnt + sb);
    float v[kItems];
    double g[kItems], h[kItems];
    int cnt[kItems];
    unsigned vm = 0;
    float vnext = 0.f;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      v[k] = 0.f; g[k] = 0.0; h[k] = 0.0;
      if (base + k < cp1) vm |= 1u << k;
    }
    if (vm) {
      if (!kTotals) {
        if (kRLE) {
          rle_values(A.t.tb, c, p0, d.len, (d.jf & kDescNext) != 0, base, K, (int)(sb + K), v, vnext);
        } else {
          const float4 v0 = __ldcs(reinterpret_cast<const float4*>(A.t.val + base));
          const float4 v1 = __ldcs(reinterpret_cast<const float4*>(A.t.val + base + 4));
          v[0] = v0.x; v[1] = v0.y; v[2] = v0.z; v[3] = v0.w; v[4] = v1.x; v[5] = v1.y; v[6] = v1.z; v[7] = v1.w;
          if (base + kItems < cp1) vnext = __ldg(A.t.val + base + kItems);
          else if (d.jf & kDescNext) vnext = d.vnext;
        }
      }
      const double2* gi = reinterpret_cast<const double2*>(A.glist + base);
      const double2* hi2 = reinterpret_cast<const double2*>(A.hlist + base);
#pragma unroll
      for (int q = 0; q < kItems / 2; ++q) {
        const double2 x = __ldcs(gi + q);
        g[2 * q] = x.x; g[2 * q + 1] = x.y;
        if (kH) { const double2 y = __ldcs(hi2 + q); h[2 * q] = y.x; h[2 * q + 1] = y.y; }
      }
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if ((vm >> k) & 1) { if (!kH) h[k] = hess_of<HMODE>(g[k]); }
        else { g[k] = 0.0; h[k] = 0.0; }
      }
    }
    const CarryD cx = carry_load(A.carry + 5ll * c);
    const SVf carry = SVf{cx.g, cx.h, cx.c, 0};
    int sj[kItems];
    unsigned hm, pem, rem;
    assign_segments<!kTotals>(ss, sc, cp1, K, base, vm, v, vnext, sj, hm, pem, rem);
    SVf run = svf_zero();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if ((vm >> k) & 1) {
        if ((hm >> k) & 1) { run.g = g[k]; run.h = h[k]; run.c = 1; run.f = 1; }
        else { run.g = run.g + g[k]; run.h = run.h + h[k]; run.c += 1; }
      }
      g[k] = run.g; h[k] = run.h; cnt[k] = run.c;
    }
    SVf inc = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const SVf y = shfl_up(inc, o);
      if (lane >= o) inc = comb(y, inc);
    }
    SVf exc = shfl_up(inc, 1);
    if (lane == 0) exc = svf_zero();
    {
      const SVf car = comb(carry, exc);
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        const bool head_before = (hm & ((2u << k) - 1u)) != 0u;
        if (!head_before) { g[k] = car.g + g[k]; h[k] = car.h + h[k]; cnt[k] = car.c + cnt[k]; }
      }
    }
    if (kTotals) {
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (((vm & rem) >> k) & 1) {
          const long long s = sb + sj[k];
          A.segPG_out[s] = g[k];
          A.segPH_out[s] = h[k];
        }
      }
      continue;
    }
    // Eq. 2 at run ends, both default directions when the segment has missing values; ranked by
    // the score, exact Eq. 2 for each segment's winner.  Segment j's present totals sit in lane j.
    double lPG = 0.0, lPH = 0.0;
    if (kMissing && K <= kWarpK && lane < K) {
      lPG = A.segPG[sb + lane];
      lPH = A.segPH[sb + lane];
    }
    double gn[kItems];
    unsigned dm = 0, okm = 0;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      gn[k] = 0.0;
      const int j = sj[k];
      double PG = 0.0, PH = 0.0;
      if (kMissing && K <= kWarpK) {  // every lane takes part in the shuffles
        PG = __shfl_sync(0xffffffffu, lPG, j & 31);
        PH = __shfl_sync(0xffffffffu, lPH, j & 31);
      }
      if (!(((vm & rem) >> k) & 1)) continue;
      const NodeV nv = node_v(B, A, K, j);
      const int cL = cnt[k];
      bool ok = false;
      double best = 0.0;
      int bd = 0;
      if (cL >= 1 && nv.C - cL >= 1) { best = split_score(g[k], h[k], nv.G, nv.H, lam); ok = true; }
      if (kMissing) {
        const int cM = nv.C - (int)sc[j];
        if (cM > 0) {
          if (K > kWarpK) { PG = A.segPG[sb + j]; PH = A.segPH[sb + j]; }
          const int cL1 = cL + cM;
          if (cL1 >= 1 && nv.C - cL1 >= 1) {
            const double g1 = split_score(g[k] + (nv.G - PG), h[k] + (nv.H - PH), nv.G, nv.H, lam);
            if (!ok || g1 > best) { best = g1; bd = 1; ok = true; }
          }
        }
      }
      gn[k] = best;
      dm |= (unsigned)bd << k;
      okm |= (unsigned)ok << k;
    }
    // per-segment argmax inside the chunk: segmented max-scan over the warp of (score, position).
    // Inside a segment the candidates are distinct values in descending order, so "earlier
    // position" is R12's "larger value"; the direction tie was settled per item (low first).
    unsigned char* sfl = flg[wid];
    double lg = -INFINITY;
    int lq = INT_MAX, lf = 0;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1)) continue;
      sfl[lane * kItems + k] = 0;
      if ((hm >> k) & 1) { lg = -INFINITY; lq = INT_MAX; lf = 1; }
      if (((okm >> k) & 1) && gn[k] > lg) { lg = gn[k]; lq = lane * kItems + k; }
    }
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const double yg = __shfl_up_sync(0xffffffffu, lg, o);
      const int yq = __shfl_up_sync(0xffffffffu, lq, o), yf = __shfl_up_sync(0xffffffffu, lf, o);
      if (lane >= o) {
        if (!lf && (yg > lg || (yg == lg && yq < lq))) { lg = yg; lq = yq; }
        lf |= yf;
      }
    }
    double cg_ = __shfl_up_sync(0xffffffffu, lg, 1);
    int cq = __shfl_up_sync(0xffffffffu, lq, 1);
    if (lane == 0) { cg_ = -INFINITY; cq = INT_MAX; }
    __syncwarp();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1)) continue;
      if ((hm >> k) & 1) { cg_ = -INFINITY; cq = INT_MAX; }
      if (((okm >> k) & 1) && gn[k] > cg_) { cg_ = gn[k]; cq = lane * kItems + k; }
      if (((pem >> k) & 1) && cq != INT_MAX) sfl[cq] = 1;  // each segment marks one item
    }
    __syncwarp();
#if GBDT_GEN_COMPACT
    // the marked items (a few per warp) through one copy of the record code: the eight unrolled
    // copies of the exact Eq. 2 (two IEEE divisions each) made the kernel overflow the
    // instruction cache (35 % of stall samples on instruction fetch, C4a)
    unsigned pmk = 0;
#pragma unroll
    for (int k = 0; k < kItems; ++k)
      if (((vm >> k) & 1) && sfl[lane * kItems + k]) pmk |= 1u << k;
    while (pmk) {
      const int k = __ffs(pmk) - 1;
      pmk &= pmk - 1;
      double gq = g[0], hq = h[0];
      int cq2 = cnt[0], j = sj[0];
      float vq = v[0];
#pragma unroll
      for (int t = 1; t < kItems; ++t)
        if (k == t) { gq = g[t]; hq = h[t]; cq2 = cnt[t]; j = sj[t]; vq = v[t]; }
      const long long s = sb + j;
      const NodeV nv = node_v(B, A, K, j);
      Rec r;
      r.value = vq;
      r.attr = A.t.a_base + d.a;
      r.dir = (dm >> k) & 1;
      r.node = j;
      r.epoch = epoch;
      r.shard = A.shard;
      r.pos = base + k;
      if (r.dir) {
        r.GL = gq + (nv.G - A.segPG[s]);
        r.HL = hq + (nv.H - A.segPH[s]);
        r.cntL = cq2 + (nv.C - (int)sc[j]);
      } else {
        r.GL = gq; r.HL = hq; r.cntL = cq2;
      }
#else
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1) || !sfl[lane * kItems + k]) continue;
      const int j = sj[k];
      const long long s = sb + j;
      const NodeV nv = node_v(B, A, K, j);
      Rec r;
      r.value = v[k];
      r.attr = A.t.a_base + d.a;
      r.dir = (dm >> k) & 1;
      r.node = j;
      r.epoch = epoch;
      r.shard = A.shard;
      r.pos = base + k;
      if (r.dir) {
        r.GL = g[k] + (nv.G - A.segPG[s]);
        r.HL = h[k] + (nv.H - A.segPH[s]);
        r.cntL = cnt[k] + (nv.C - (int)sc[j]);
      } else {
        r.GL = g[k]; r.HL = h[k]; r.cntL = cnt[k];
      }
#endif
      r.gain = eq2_gain(r.GL, r.HL, nv.G, nv.H, lam, nv.P);
      if (K <= kWarpK) {
        const unsigned long long gk = gain_key(r.gain);
        if (rec_better(gk, r, wgk[wid][j], wrec[wid][j])) { wgk[wid][j] = gk; wrec[wid][j] = r; }
      } else {
        post_global(A, r);
      }
    }
    __syncwarp();
    }
  }
  if (!kTotals && K <= kWarpK) merge_warp_tables(A, K, wgk, wrec);  // one record per node and CTA
}

// ============================================================================ a8: partition
// One warp per chunk: (high, low) entry counts (packed hi | lo << 32) + reset flag; with missing
// values also the per-segment counts (the plan needs them).
// Short chunk of k_part_count (<= 32 entries, K <= 32, per-segment counts wanted): lane i on
// entry p0 + i, side counts by ballots over the lanes, one atomic pair per segment piece (the
// piece's last lane), the side-list written in the same 4-entry words.  The ids were streamed into
// L1/L2 by the warp's prefetch, so the reload here hits.
__device__ __forceinline__ void count_short(const PartArgs& A, const ChunkMeta& M, int c, int K, int lane) {
  const long long p0 = M.p0;
  const int len = (int)(M.p1 - p0);
  const bool valid = lane < len;
  const long long p = p0 + lane;
  unsigned sd = 0;
  if (valid) sd = __ldg(A.side + __ldg(A.t.ins + p));
  const unsigned bh = __ballot_sync(0xffffffffu, sd == 1), bl = __ballot_sync(0xffffffffu, sd == 2);
  // side-list words: lane 4q packs lanes 4q .. 4q+3 (invalid lanes hold 0, as in the general path)
  unsigned w = sd;
  w |= __shfl_down_sync(0xffffffffu, sd, 1) << 8;
  w |= __shfl_down_sync(0xffffffffu, sd, 2) << 16;
  w |= __shfl_down_sync(0xffffffffu, sd, 3) << 24;
  if ((lane & 3) == 0 && valid) reinterpret_cast<unsigned*>(A.slist + p)[0] = w;
  // segment pieces (as in sf_short): heads from the attribute's segment table, one segment per lane
  const long long* ss = (const long long*)(A.t.tb.seg_start + M.sb);
  const long long* sc = (const long long*)(A.t.tb.seg_cnt + M.sb);
  const long long s_l = lane < K ? ss[lane] : LLONG_MAX;
  const long long c_l = lane < K ? sc[lane] : 0;
  const unsigned le0 = __ballot_sync(0xffffffffu, s_l <= p0);
  const int j0 = 31 - __clz(le0 | 1u);
  const bool starts = lane < K && c_l > 0 && s_l >= p0 && s_l < p0 + len;
  const unsigned hm = __reduce_or_sync(0xffffffffu, starts ? (1u << (int)(s_l - p0)) : 0u);
  const unsigned upto = hm & (0xffffffffu >> (31 - lane));
  const int hpos = upto ? 31 - __clz(upto) : -1;
  int j = j0;
  unsigned o = __ballot_sync(0xffffffffu, starts);
  while (o) {
    const int l = __ffs(o) - 1;
    o &= o - 1;
    const long long sll = __shfl_sync(0xffffffffu, s_l, l);
    if (hpos >= 0 && sll - p0 == hpos) j = l;
  }
  const bool piece_end = valid && (lane == len - 1 || ((hm >> (lane + 1)) & 1u));
  if (piece_end) {
    const int sl = hpos >= 0 ? hpos : 0;
    const unsigned pm = (0xffffffffu >> (31 - lane)) & (0xffffffffu << sl);
    const int ch = __popc(bh & pm), cl = __popc(bl & pm);
    if (ch) atomicAdd(A.segH + M.sb + j, ch);
    if (cl) atomicAdd(A.segL + M.sb + j, cl);
  }
  if (lane == 0) {
    A.ccnt[2ll * c] = (unsigned long long)__popc(bh) | ((unsigned long long)__popc(bl) << 32);
    A.ccnt[2ll * c + 1] = (unsigned long long)M.reset;
  }
}

#ifndef GBDT_COUNT_SHORT
#define GBDT_COUNT_SHORT 1
#endif
#ifndef GBDT_COUNT_CTAS
#define GBDT_COUNT_CTAS 0  // 0: the compiler's choice (a minimum of 1 CTA/SM would let it take more registers)
#endif
#if GBDT_COUNT_CTAS > 0
#define LB_GBDT_COUNT_CTAS __launch_bounds__(kThreads, GBDT_COUNT_CTAS)
#else
#define LB_GBDT_COUNT_CTAS __launch_bounds__(kThreads)
#endif
__global__ void LB_GBDT_COUNT_CTAS k_part_count(PartArgs A, int counted) {
  __shared__ TabCache tc;
  const int lane = threadIdx.x & 31;
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0 || C == 0) return;
  tab_load(tc, A.t);
  __syncthreads();
  const int nw = (gridDim.x * blockDim.x) >> 5;
  // software pipeline: the instance ids of the warp's next chunk are loaded before the side
  // gathers of the current one, so the list stream and the (L2) gathers overlap
  const int NC = nchunks(A.t.tb);
  int i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  int4 n0 = make_int4(0, 0, 0, 0), n1 = n0;
  auto load_ids = [&](int cc, int4& a0, int4& a1) {
    const ChunkMeta Mx = chunk_meta(tc, A.t, K, cc);
    const long long b = Mx.p0 + (long long)lane * kItems;
    if (b < Mx.p1) {
      a0 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + b));
      if (b + 4 < Mx.p1) a1 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + b + 4));
    }
  };
  if (i < NC) load_ids(chunk_at(A.t.tb, i), n0, n1);
  for (; i < NC; i += nw) {
    const int c = chunk_at(A.t.tb, i);
    const ChunkMeta M = chunk_meta(tc, A.t, K, c);
    const long long base = M.p0 + (long long)lane * kItems;
    const int4 i0 = n0, i1 = n1;
    if (i + nw < NC) load_ids(chunk_at(A.t.tb, i + nw), n0, n1);
#if GBDT_COUNT_SHORT
    if (counted && M.p1 - M.p0 <= 32 && K <= 32) {
      count_short(A, M, c, K, lane);
      continue;
    }
#endif
    unsigned vm = 0, loc = 0;
    uint8_t sd[kItems];
#pragma unroll
    for (int k = 0; k < kItems; ++k) sd[k] = 0;
    if (base < M.p1) {
      const int id[kItems] = {i0.x, i0.y, i0.z, i0.w, i1.x, i1.y, i1.z, i1.w};
#pragma unroll
      for (int k = 0; k < kItems; ++k)
        if (base + k < M.p1) { vm |= 1u << k; sd[k] = __ldg(A.side + id[k]); }
#pragma unroll
      for (int k = 0; k < kItems; ++k) loc += sd[k] == 1 ? 1u : (sd[k] == 2 ? (1u << 16) : 0u);
      // the entry-aligned side-list lets the scatter stream sides instead of gathering again
      // (4-entry granules: lists are padded to 4 entries, so never write past this list)
      unsigned w0 = 0, w1 = 0;
#pragma unroll
      for (int k = 0; k < 4; ++k) { w0 |= (unsigned)sd[k] << (8 * k); w1 |= (unsigned)sd[k + 4] << (8 * k); }
      reinterpret_cast<unsigned*>(A.slist + base)[0] = w0;
      if (base + 4 < M.p1) reinterpret_cast<unsigned*>(A.slist + base)[1] = w1;
    }
    if (counted && vm) {
      int sj[kItems];
      unsigned hm, pem, rem;
      float vd[kItems];
      assign_segments<false>((const long long*)(A.t.tb.seg_start + M.sb), (const long long*)(A.t.tb.seg_cnt + M.sb),
                             M.p1, K, base, vm, vd, 0.f, sj, hm, pem, rem);
      int cur = -1, ch = 0, cl = 0;
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (!((vm >> k) & 1)) continue;
        if (sj[k] != cur) {
          if (cur >= 0) {
            if (ch) atomicAdd(A.segH + M.sb + cur, ch);
            if (cl) atomicAdd(A.segL + M.sb + cur, cl);
          }
          cur = sj[k]; ch = cl = 0;
        }
        ch += sd[k] == 1;
        cl += sd[k] == 2;
      }
      if (cur >= 0) {
        if (ch) atomicAdd(A.segH + M.sb + cur, ch);
        if (cl) atomicAdd(A.segL + M.sb + cur, cl);
      }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) loc += __shfl_xor_sync(0xffffffffu, loc, o);
    if (lane == 0) {
      A.ccnt[2ll * c] = (unsigned long long)(loc & 0xffffu) | ((unsigned long long)(loc >> 16) << 32);
      A.ccnt[2ll * c + 1] = (unsigned long long)M.reset;
    }
  }
}

// Dense variant (no per-segment counts needed): two chunks per warp iteration in the striped
// arrangement, so 16 instance-id loads and then 16 side gathers per lane are in flight at once;
// the side gathers ask L2 to keep the per-instance side array (evict-last) while the lists stream
// past it.  Counts by ballot; the side-list rows are written as coalesced 32-byte rows.
__device__ __forceinline__ uint8_t ld_keep_u8(const uint8_t* p, unsigned long long pol) {
  unsigned short v;
  asm volatile("ld.global.nc.L2::cache_hint.u8 %0, [%1], %2;" : "=h"(v) : "l"(p), "l"(pol));
  return (uint8_t)v;
}
__device__ __forceinline__ unsigned ld_keep_u32(const uint32_t* p, unsigned long long pol) {
  unsigned v;
  asm volatile("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(p), "l"(pol));
  return v;
}
#ifndef GBDT_CDENSE_CTAS
#define GBDT_CDENSE_CTAS 0  // 0: the compiler's choice (a minimum of 1 CTA/SM would let it take more registers)
#endif
#if GBDT_CDENSE_CTAS > 0
#define LB_GBDT_CDENSE_CTAS __launch_bounds__(kThreads, GBDT_CDENSE_CTAS)
#else
#define LB_GBDT_CDENSE_CTAS __launch_bounds__(kThreads)
#endif
__global__ void LB_GBDT_CDENSE_CTAS k_part_count_dense(PartArgs A) {
  __shared__ TabCache tc;
  const int lane = threadIdx.x & 31;
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0 || C == 0) return;
  tab_load(tc, A.t);
  __syncthreads();
  const unsigned long long keep = policy_evict_last();
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < C; c += 2 * nw) {
    long long p0[2];
    int len[2], rs[2], id[2][kItems], mode[2];
    uint8_t sd[2][kItems];
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const int cu = c + u * nw;
      len[u] = 0;
      p0[u] = 0;
      rs[u] = 0;
      mode[u] = 0;
      if (cu < C) {
        const ChunkMeta M = chunk_meta(tc, A.t, K, cu);
        p0[u] = M.p0;
        len[u] = (int)(M.p1 - M.p0);
        rs[u] = M.reset;
        // a chunk inside one segment: nothing to gather if its node became a leaf, else one bit
        // per entry from the 1.4 MB high-child bitmap; a chunk crossing segments: side bytes
        const SegOf sg = warp_seg((const long long*)(A.t.tb.seg_start + M.sb),
                                  (const long long*)(A.t.tb.seg_cnt + M.sb), K, M.p0, lane);
        mode[u] = M.p1 <= sg.se ? (A.cidx[sg.j] < 0 ? 0 : 1) : 2;
      }
      const int32_t* ip = A.t.ins + p0[u] + lane;
#pragma unroll
      for (int k = 0; k < kItems; ++k) id[u][k] = (32 * k + lane < len[u] && mode[u]) ? __ldcs(ip + 32 * k) : -1;
    }
#pragma unroll
    for (int u = 0; u < 2; ++u)
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        uint8_t x = 0;
        if (id[u][k] >= 0) {
          if (mode[u] == 1) x = ((ld_keep_u32(A.hbit + (id[u][k] >> 5), keep) >> (id[u][k] & 31)) & 1u) ? 1 : 2;
          else x = ld_keep_u8(A.side + id[u][k], keep);
        }
        sd[u][k] = x;
      }
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const int cu = c + u * nw;
      if (cu >= C) break;
      unsigned nh = 0, nl = 0;
      uint8_t* so = A.slist + p0[u] + lane;
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        nh += __popc(__ballot_sync(0xffffffffu, sd[u][k] == 1));
        nl += __popc(__ballot_sync(0xffffffffu, sd[u][k] == 2));
        if (32 * k + lane < len[u]) __stcs(so + 32 * k, sd[u][k]);
      }
      if (lane == 0) {
        A.ccnt[2ll * cu] = (unsigned long long)nh | ((unsigned long long)nl << 32);
        A.ccnt[2ll * cu + 1] = (unsigned long long)rs[u];
      }
    }
  }
}

__device__ unsigned long long block_exscan_u64(unsigned long long x, unsigned long long& total) {
  __shared__ unsigned long long ws[32];
  __shared__ unsigned long long tot;
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
  if (threadIdx.x == blockDim.x - 1) tot = ex + x;
  __syncthreads();
  total = tot;
  __syncthreads();
  return ex;
}

// Child placement (stable, attribute-major, children in heap order) and the next level's
// attribute / chunk / segment tables, attribute-parallel:
//   k_plan_attr  per attribute: (high, low) counts before each segment and the child list length
//   (exact integer scan over the attributes of (padded length | chunks << 32))
//   k_plan_seg   per attribute: list start, chunk start, every child segment's start and count
// A group of G lanes per attribute (G = K rounded up to a power of two, at most 32; tiles of 32
// segments when K > 32), lane j of the group on segment j: the segment tables are read and written
// in coalesced rows, all lanes busy whatever K, and the running offsets are group scans.  (A thread
// per attribute looping over its K segments strided every write by K words: on C4a, 1.35 M
// attributes x up to 32 segments, k_plan_seg moved 3x its algorithmic bytes in partial sectors.)
__device__ __forceinline__ int plan_group(int K) {
  int G = 1;
  while (G < K && G < 32) G <<= 1;
  return G;
}

__global__ void __launch_bounds__(kThreads) k_plan_attr(PlanArgs A) {
  const int K = *A.Kp, m = A.m;
  const int lane = threadIdx.x & 31;
  const int G = plan_group(K), per = 32 / G, sub = lane / G, jj = lane % G;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int a0 = ((blockIdx.x * blockDim.x + threadIdx.x) >> 5) * per; a0 <= m; a0 += nw * per) {
    const int a = a0 + sub;
    // in-place short lists take no room in the level buffers and have no segments
    const bool skip = a < m && A.inplace && A.sflag && A.sflag[a];
    const bool act = a < m && !skip;
    if (a == m && jj == 0) { A.el[2ll * m] = 0ull; A.el[2ll * m + 1] = 0ull; }
    unsigned long long pre = 0;
    long long L = 0;
    for (int j0 = 0; j0 < K; j0 += G) {
      const int j = j0 + jj;
      const long long s = (long long)a * K + j;
      unsigned long long x = 0;
      long long l = 0;
      if (act && j < K) {
        const int c = A.cidx[j];
        unsigned hi, lo;
        if (!A.counted) {  // no missing values: every instance of a node is in every attribute list
          hi = c >= 0 ? (unsigned)A.ncnt[c] : 0u;
          lo = c >= 0 ? (unsigned)A.ncnt[c + 1] : 0u;
          A.segH[s] = (int32_t)hi;
          A.segL[s] = (int32_t)lo;
        } else {
          hi = (unsigned)A.segH[s];
          lo = (unsigned)A.segL[s];
        }
        x = (unsigned long long)hi | ((unsigned long long)lo << 32);
        if (c >= 0) l = (long long)hi + lo;
      }
      unsigned long long inc = x;
      for (int o = 1; o < G; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(0xffffffffu, inc, o, G);
        if (jj >= o) inc += y;
      }
      if (act && j < K) A.seg_pre[s] = pre + (inc - x);
      pre += __shfl_sync(0xffffffffu, inc, G - 1, G);
      for (int o = G >> 1; o; o >>= 1) l += __shfl_xor_sync(0xffffffffu, l, o, G);
      L += l;
    }
    if ((act || skip) && jj == 0) {
      A.nxt.col_len[a] = L;
      A.el[2ll * a] = (unsigned long long)((L + 3) & ~3ll) | ((unsigned long long)((L + kChunk - 1) / kChunk) << 32);
      A.el[2ll * a + 1] = 0ull;
    }
  }
}

__global__ void __launch_bounds__(kThreads) k_plan_seg(PlanArgs A) {
  const int K = *A.Kp, Kn = *A.Knp, m = A.m;
  const int lane = threadIdx.x & 31;
  const int G = plan_group(K), per = 32 / G, sub = lane / G, jj = lane % G;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int a0 = ((blockIdx.x * blockDim.x + threadIdx.x) >> 5) * per; a0 <= m; a0 += nw * per) {
    const int a = a0 + sub;
    const bool act = a < m && !(A.inplace && A.sflag && A.sflag[a]);  // (in-place short lists: no segments)
    long long cs = 0;
    if (a <= m) {
      const unsigned long long ex = A.el[2ll * a];
      cs = (long long)(ex & 0xffffffffull);
      const int ch = (int)(ex >> 32);
      if (jj == 0) {
        A.nxt.col_start[a] = cs;
        A.nxt.chunk_start[a] = ch;
        if (a == m) {
          *A.nxt.C = ch;
          *A.nxt.T = (ch + kChunksPerTile - 1) / kChunksPerTile;
          if (A.nxt.nlc) *A.nxt.nlc = 0;  // k_chunk_attr lists the chunk kernels' chunks
        }
      }
    }
    long long r = cs;
    for (int j0 = 0; j0 < K; j0 += G) {
      const int j = j0 + jj;
      const int c = (act && j < K) ? A.cidx[j] : -1;
      const long long s = (long long)a * K + j;
      long long hi = 0, lo = 0;
      if (c >= 0) { hi = A.segH[s]; lo = A.segL[s]; }
      const long long x = hi + lo;
      long long inc = x;
      for (int o = 1; o < G; o <<= 1) {
        const long long y = __shfl_up_sync(0xffffffffu, inc, o, G);
        if (jj >= o) inc += y;
      }
      if (c >= 0) {
        const long long st = r + (inc - x);
        const long long sn = (long long)a * Kn + c;
        A.out_hi[s] = st;
        A.nxt.seg_start[sn] = st;
        A.nxt.seg_cnt[sn] = hi;
        A.out_lo[s] = st + hi;
        A.nxt.seg_start[sn + 1] = st + hi;
        A.nxt.seg_cnt[sn + 1] = lo;
      }
      r += __shfl_sync(0xffffffffu, inc, G - 1, G);
    }
  }
}

// attribute of every chunk of the next level (the largest a with chunk_start[a] <= c)
// and, on the short path, the list of the chunk kernels' chunks: those of the other attributes
// (every chunk when K' > 32, where the short kernels stand down)
__global__ void __launch_bounds__(kThreads) k_chunk_attr(PlanArgs A) {
  const int C = *A.nxt.C, m = A.m;
  const int lane = threadIdx.x & 31;
  const bool sp = A.nxt.lc && A.sflag && *A.Knp <= 32;
  for (int c0 = (blockIdx.x * blockDim.x + threadIdx.x) - lane; c0 < C; c0 += gridDim.x * blockDim.x) {
    const int c = c0 + lane;
    int a = 0;
    if (c < C) {
      a = find_attr(A.nxt.chunk_start, m, c);
      A.nxt.chunk_attr[c] = a;
    }
    if (A.nxt.lc) {  // warp-aggregated append, chunk order kept inside the warp
      const bool keep = c < C && !(sp && A.sflag[a]);
      const unsigned b = __ballot_sync(0xffffffffu, keep);
      int base = 0;
      if (lane == 0 && b) base = atomicAdd(A.nxt.nlc, __popc(b));
      base = __shfl_sync(0xffffffffu, base, 0);
      if (keep) A.nxt.lc[base + __popc(b & ((1u << lane) - 1u))] = c;
    }
  }
}

// Stable scatter ("Scatter"), one warp per chunk: out(e) = out_base(seg, side) + rank of
// e among the segment's same-side entries = C_side(e) - C_side(seg start), C counted within the
// attribute (chunk prefix from the count scan + in-chunk exclusive count).  The chunk is read in
// the STRIPED arrangement (item k of lane l is entry p0 + 32 k + l): every load is one coalesced
// row, and within a row the kept entries of one side are ranked by a ballot, so consecutive lanes
// write consecutive destinations straight from registers (no staging, no bank conflicts).
// g (h) move along with the entries.
// Exact fixed-point add of v into the 128-bit record word pair p[0] (lo), p[1] (hi): the low word's
// carry is propagated by this contribution itself, so the total is exact in any order.
__device__ __forceinline__ void fx_atomic_add(unsigned long long* p, __int128 v) {
  const unsigned long long lo = (unsigned long long)v, hi = (unsigned long long)((unsigned __int128)v >> 64);
  const unsigned long long old = atomicAdd(p, lo);
  const unsigned long long c = (old + lo < old) ? 1ull : 0ull;
  if (hi + c) atomicAdd(p + 1, hi + c);
}

// Does an entry of the child segment ending at child_end count in the segmented aggregate of the
// next-level chunk x (attribute list [cs, ce))?  Yes iff no non-empty segment starts after it in
// the chunk, i.e. the child reaches the chunk's end (or the end of the list).
__device__ __forceinline__ bool agg_counts(long long child_end, long long cs, long long ce, long long xi) {
  return child_end >= min(cs + ((xi + 1) << 8), ce);
}

// Sum of v[0..7] over the warp, transpose-reduced: afterwards lane l holds the total of value
// ((l >> 2) & 7) (bit-reversed grouping below), so lanes 0, 4, ..., 28 hold the eight totals.
__device__ __forceinline__ double warp_sum8(double (&v)[8], int lane) {
  const bool u16 = lane & 16, u8 = lane & 8, u4 = lane & 4;
  double w4[4], w2[2];
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    const double send = u16 ? v[i] : v[i + 4], keep = u16 ? v[i + 4] : v[i];
    w4[i] = keep + __shfl_xor_sync(0xffffffffu, send, 16);
  }
#pragma unroll
  for (int i = 0; i < 2; ++i) {
    const double send = u8 ? w4[i] : w4[i + 2], keep = u8 ? w4[i + 2] : w4[i];
    w2[i] = keep + __shfl_xor_sync(0xffffffffu, send, 8);
  }
  double w = (u4 ? w2[1] : w2[0]) + __shfl_xor_sync(0xffffffffu, u4 ? w2[0] : w2[1], 4);
  w += __shfl_xor_sync(0xffffffffu, w, 2);
  w += __shfl_xor_sync(0xffffffffu, w, 1);
  return w;  // value index (u16 ? 4 : 0) + (u8 ? 2 : 0) + (u4 ? 1 : 0)
}

template <int HMODE, bool kRLE, bool kAgg>
#ifndef GBDT_SCATTER_CTAS
#define GBDT_SCATTER_CTAS 3
#endif
#ifndef GBDT_SCATTER_ROWS
#define GBDT_SCATTER_ROWS 4
#endif
#ifndef GBDT_SCATTER_STCS
#define GBDT_SCATTER_STCS 1  // evict-first stores: 11.76 -> 11.38 ms/tree of scatter on C3
#endif
__global__ void __launch_bounds__(kThreads, GBDT_SCATTER_CTAS) k_part_scatter(PartArgs A) {
  constexpr bool kH = HMODE == kHGather;
  constexpr int kHalf = GBDT_SCATTER_ROWS;  // rows loaded per step
  __shared__ TabCache tc;
  __shared__ long long wss[kWarps][kWarpK];  // the attribute's segment starts (chunks crossing segments)
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0 || C == 0) return;
  const int Fg = kAgg ? A.fx[0] : 0, Fh = kAgg ? A.fx[1] : 0;
  tab_load(tc, A.t);
  __syncthreads();
  const unsigned lt = (1u << lane) - 1u;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  const int NC = nchunks(A.t.tb);
  for (int i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < NC; i += nw) {
    const int c = chunk_at(A.t.tb, i);
    const ChunkMeta M = chunk_meta(tc, A.t, K, c);
    const long long p0 = M.p0;
    const int len = (int)(M.p1 - p0);
    if (i + nw < NC) {  // the warp's next chunk streams into L2 meanwhile
      const long long pn = chunk_meta(tc, A.t, K, chunk_at(A.t.tb, i + nw)).p0;
      prefetch_chunk(A.t.ins, pn, 4, lane);
      prefetch_chunk(A.g_in, pn, 8, lane);
      if (!kRLE) prefetch_chunk(A.t.val, pn, 4, lane);
      if (kH) prefetch_chunk(A.h_in, pn, 8, lane);
    }
    // chunk-relative lane pointers (item k of the lane is entry p0 + 32 k + lane)
    const uint8_t* sp_ = A.slist + p0 + lane;
    const int32_t* ip_ = A.t.ins + p0 + lane;
    const float* vp_ = A.t.val + p0 + lane;
    const double* gp_ = A.g_in + p0 + lane;
    const double* hp_ = A.h_in + p0 + lane;
    const long long* ss = (const long long*)(A.t.tb.seg_start + M.sb);
    const long long* scn = (const long long*)(A.t.tb.seg_cnt + M.sb);
    const SegOf sg = warp_seg(ss, scn, K, p0, lane);
    const bool single = M.p1 <= sg.se;  // warp-uniform; nearly always on dense data
    const unsigned long long cpv = A.cpre[2ll * c];
    const long long chi0 = (long long)(cpv & 0xffffffffull), clo0 = (long long)(cpv >> 32);
    long long dh0 = 0, dl0 = 0, ehi = 0, elo = 0;
    if (single) {
      const long long s = M.sb + sg.j;
      const unsigned long long sp = A.seg_pre[s];
      const long long oh = A.out_hi[s], ol = A.out_lo[s];
      dh0 = oh + chi0 - (long long)(sp & 0xffffffffull);
      dl0 = ol + clo0 - (long long)(sp >> 32);
      if (kAgg) { ehi = oh + A.segH[s]; elo = ol + A.segL[s]; }  // ends of the two child segments
    } else if (K <= kWarpK) {
      if (lane < K) wss[wid][lane] = ss[lane];
      __syncwarp();
    }
    // next level: the attribute's list and chunk origin; entries of each side before the
    // destination chunk boundary that follows the side's first destination
    long long ncs = 0, nce = 0;
    int ncb = 0, cutH = 0, cutL = 0;
    if (kAgg) {
      ncs = A.nxt.col_start[M.a];
      nce = ncs + A.nxt.col_len[M.a];
      ncb = A.nxt.chunk_start[M.a];
      cutH = kChunk - (int)((dh0 - ncs) & (kChunk - 1));
      cutL = kChunk - (int)((dl0 - ncs) & (kChunk - 1));
    }
    double acc[8];  // (high A, high B, low A, low B) x (g, h); A: before the boundary
#pragma unroll
    for (int i = 0; i < 8; ++i) acc[i] = 0.0;
    int nh = 0, nl = 0;  // kept entries of each side in the rows before
#pragma unroll
    for (int half = 0; half < kItems / kHalf; ++half) {
      if (half > 0 && 32 * half * kHalf >= len) break;  // short lists: no empty rows (warp-uniform)
      uint8_t sd[kHalf];
      int id[kHalf];
      float v[kHalf];
      double g[kHalf], h[kHalf];
#pragma unroll
      for (int kk = 0; kk < kHalf; ++kk) {
        const int o = 32 * (half * kHalf + kk);
        sd[kk] = 0; id[kk] = 0; v[kk] = 0.f; g[kk] = 0.0; h[kk] = 0.0;
        if (o + lane < len) {
          sd[kk] = __ldcs(sp_ + o);
          id[kk] = __ldcs(ip_ + o);
          if (!kRLE) v[kk] = __ldcs(vp_ + o);  // with RLE the values live in the runs
          g[kk] = __ldcs(gp_ + o);
          if (kH) h[kk] = __ldcs(hp_ + o);
        }
      }
#pragma unroll
      for (int kk = 0; kk < kHalf; ++kk) {
        const int k = half * kHalf + kk;
        if (kk > 0 && 32 * k >= len) break;
        const unsigned bh = __ballot_sync(0xffffffffu, sd[kk] == 1), bl = __ballot_sync(0xffffffffu, sd[kk] == 2);
        if (sd[kk]) {
          const bool hi = sd[kk] == 1;
          const int rk = hi ? nh + __popc(bh & lt) : nl + __popc(bl & lt);
          long long d;
          if (single) {
            d = (hi ? dh0 : dl0) + rk;
            if (kAgg) {
              const double hk = kH ? h[kk] : hess_of<HMODE>(g[kk]);
              const int slot = (hi ? 0 : 4) + (rk < (hi ? cutH : cutL) ? 0 : 2);
#pragma unroll
              for (int i = 0; i < 8; i += 2)
                if (slot == i) { acc[i] += g[kk]; acc[i + 1] += hk; }
            }
          } else {
            const long long p = p0 + 32 * k + lane;
            int lo = 0, hi2 = K - 1;  // largest j with ss[j] <= p
            while (lo < hi2) {
              const int mid = (lo + hi2 + 1) >> 1;
              if ((K <= kWarpK ? wss[wid][mid] : ss[mid]) <= p) lo = mid; else hi2 = mid - 1;
            }
            const long long s = M.sb + lo;
            const unsigned long long sp = A.seg_pre[s];
            d = hi ? A.out_hi[s] + (chi0 + rk - (long long)(sp & 0xffffffffull))
                   : A.out_lo[s] + (clo0 + rk - (long long)(sp >> 32));
            if (kAgg) {  // rare (chunks crossing segments): the entry's own exact contribution
              const double hk = kH ? h[kk] : hess_of<HMODE>(g[kk]);
              const long long xi = (d - ncs) >> 8;
              const long long cend = hi ? A.out_hi[s] + A.segH[s] : A.out_lo[s] + A.segL[s];
              if (agg_counts(cend, ncs, nce, xi)) {
                unsigned long long* rec = A.cagg_next + 5ll * (ncb + xi);
                fx_atomic_add(rec, to_fx(g[kk], Fg));
                fx_atomic_add(rec + 2, to_fx(hk, Fh));
              }
            }
          }
#if GBDT_SCATTER_STCS
          if (!kRLE) __stcs(A.val_out + d, v[kk]);
          __stcs(A.ins_out + d, id[kk]);
          __stcs(A.g_out + d, g[kk]);
          if (kH) __stcs(A.h_out + d, h[kk]);
#else
          if (!kRLE) A.val_out[d] = v[kk];
          A.ins_out[d] = id[kk];
          A.g_out[d] = g[kk];
          if (kH) A.h_out[d] = h[kk];
#endif
        }
        nh += __popc(bh);
        nl += __popc(bl);
      }
    }
    if (kAgg && single) {
      // warp totals of the four (side, destination chunk) parts, then one exact atomic add each
      const double tot = warp_sum8(acc, lane);
      const int vi = ((lane & 16) ? 4 : 0) + ((lane & 8) ? 2 : 0) + ((lane & 4) ? 1 : 0);
      if ((lane & 3) == 0) {
        const bool hiS = vi < 4, B = (vi >> 1) & 1, isH = vi & 1;
        const int n = hiS ? nh : nl, cut = hiS ? cutH : cutL;
        const int cnt = B ? n - min(n, cut) : min(n, cut);
        const long long d0 = hiS ? dh0 : dl0;
        const long long xi = ((d0 - ncs) >> 8) + (B ? 1 : 0);
        if (cnt > 0 && agg_counts(hiS ? ehi : elo, ncs, nce, xi))
          fx_atomic_add(A.cagg_next + 5ll * (ncb + xi) + (isH ? 2 : 0), to_fx(tot, isH ? Fh : Fg));
      }
    }
    if (!single) __syncwarp();  // wss is rewritten by the warp's next crossing chunk
  }
}

// Chunk descriptors and scan flags of a level whose chunk aggregates the previous scatter
// accumulated (no missing values), one thread per chunk: the same descriptor k_chunk_agg writes,
// and word 4 of the aggregate record: entries after the chunk's last segment head (all of them
// when there is none) | head-inside << 32 | first-chunk-of-attribute << 33.
__global__ void __launch_bounds__(kThreads) k_desc(SplitArgs A) {
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0) return;
  for (int c = blockIdx.x * blockDim.x + threadIdx.x; c < C; c += gridDim.x * blockDim.x) {
    const int a = A.t.tb.chunk_attr[c];
    const long long cs = A.t.tb.col_start[a], cl = A.t.tb.col_len[a];
    const int k = c - A.t.tb.chunk_start[a];
    const long long p0 = cs + (long long)k * kChunk, p1 = min(p0 + (long long)kChunk, cs + cl);
    const bool more = p1 < cs + cl;
    const long long* ss = (const long long*)(A.t.tb.seg_start + (long long)a * K);
    const long long* sc = (const long long*)(A.t.tb.seg_cnt + (long long)a * K);
    int lo = 0, hi = K - 1;  // largest j with ss[j] <= p0
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (ss[mid] <= p0) lo = mid; else hi = mid - 1;
    }
    const int j0 = lo;
    const long long s0 = ss[j0], se = s0 + sc[j0];
    const bool single = p1 <= se;
    lo = j0; hi = K - 1;  // largest j with ss[j] < p1, then back over empty segments
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (ss[mid] < p1) lo = mid; else hi = mid - 1;
    }
    int j1 = lo;
    while (j1 > 0 && sc[j1] == 0 && ss[j1] >= p0) --j1;
    const bool head = sc[j1] > 0 && ss[j1] >= p0 && ss[j1] < p1;
    const long long cnt = head ? p1 - ss[j1] : p1 - p0;
    ChunkDesc d;
    d.p0 = p0;
    d.se = se;
    d.len = (int)(p1 - p0);
    d.a = a;
    d.jf = j0 | (s0 == p0 ? kDescHead0 : 0) | (single ? kDescSingle : 0) | (more ? kDescNext : 0);
    d.vnext = (more && !A.rle) ? A.t.val[p1] : 0.f;
    A.desc[c] = d;
    A.cagg[5ll * c + 4] = (unsigned long long)cnt | ((unsigned long long)(head ? 1 : 0) << 32) |
                          ((unsigned long long)(k == 0 ? 1 : 0) << 33);
    if (!single) A.genlist[atomicAdd(A.ngen, 1)] = c;
  }
}

// ============================================================================ a8 RLE: direct split
// "each RLE element is potentially split into two ... we compute the length of each new RLE element
// using the instance to node mapping ... prefix sum to remove the RLE element with length of 0"
// (P:250).  k_run_count: one warp per run counts its entries going high (h_r) / low (l_r) from the
// side-list.  Two exact integer scans follow: (h_r, l_r) segmented by parent segment (the child
// run's offset inside its child segment) and the non-empty flags ([h_r>0], [l_r>0]) over all runs
// (the compaction).  k_run_scatter writes the child runs -- high child of every parent segment,
// then its low child, in segment order -- and the next level's segment -> run table.
// (high | low << 32) side counts of the attribute before list position p (p inside the attribute
// list, or its end): the chunk prefix from the count scan + the warp's count inside the chunk.
__device__ __forceinline__ unsigned long long side_prefix(const RunArgs& A, int a, long long p, int lane) {
  const long long cs = A.cur.col_start[a];
  const long long k = (p - cs - 1) / kChunk;  // chunk of entry p-1 (p > cs)
  const long long q0 = cs + k * kChunk;
  const unsigned long long pre = A.cpre[2 * ((long long)A.cur.chunk_start[a] + k)];
  const long long b = q0 + lane * kItems;
  unsigned h = 0, l = 0;
  if (b < p) {
    const unsigned w0 = reinterpret_cast<const unsigned*>(A.slist + b)[0];
    const unsigned w1 = b + 4 < p ? reinterpret_cast<const unsigned*>(A.slist + b)[1] : 0u;
#pragma unroll
    for (int i = 0; i < kItems; ++i) {
      const unsigned sd = ((i < 4 ? w0 : w1) >> (8 * (i & 3))) & 0xffu;
      const bool in = b + i < p;
      h += in && sd == 1;
      l += in && sd == 2;
    }
  }
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    h += __shfl_xor_sync(0xffffffffu, h, o);
    l += __shfl_xor_sync(0xffffffffu, l, o);
  }
  return pre + ((unsigned long long)h | ((unsigned long long)l << 32));
}

__global__ void __launch_bounds__(kThreads) k_run_count(RunArgs A) {
  const int R = *A.cur.R;
  const int K = *A.Kp;
  const long long S = (long long)A.m * K;
  const int lane = threadIdx.x & 31;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  if (blockIdx.x == 0 && threadIdx.x == 0) {
    A.fl[2ll * R] = 0ull;
    A.fl[2ll * R + 1] = 0ull;
    *A.Rp1 = R + 1;
  }
  for (int r = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; r < R; r += nw) {
    long long lo = 0, hi = S - 1;  // last segment whose first run is <= r (it contains r)
    while (lo < hi) {
      const long long mid = (lo + hi + 1) >> 1;
      if (A.cur.seg_run[mid] <= r) lo = mid; else hi = mid - 1;
    }
    const long long p0 = A.cur.run_pos[r];
    const int len = A.cur.run_len[r];
    unsigned long long hl;
    if (len <= 2 * kChunk) {  // short run: count its own sides
      unsigned h = 0, l = 0;
      for (int q = lane; q < len; q += 32) {
        const uint8_t sd = A.slist[p0 + q];
        h += sd == 1;
        l += sd == 2;
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        h += __shfl_xor_sync(0xffffffffu, h, o);
        l += __shfl_xor_sync(0xffffffffu, l, o);
      }
      hl = (unsigned long long)h | ((unsigned long long)l << 32);
    } else {  // long run: difference of two attribute prefixes (work independent of the length)
      const int a = (int)(lo / K);
      hl = side_prefix(A, a, p0 + len, lane) - side_prefix(A, a, p0 + 1, lane);
      const uint8_t sd0 = A.slist[p0];  // side_prefix(p0 + 1) counted entry p0 too
      hl += (unsigned long long)(sd0 == 1) | ((unsigned long long)(sd0 == 2) << 32);
    }
    if (lane == 0) {
      const unsigned h = (unsigned)(hl & 0xffffffffull), l = (unsigned)(hl >> 32);
      A.run_seg[r] = (int32_t)lo;
      A.run_hl[r] = hl;
      A.cnt[2ll * r] = hl;
      A.cnt[2ll * r + 1] = A.cur.seg_run[lo] == r ? 1ull : 0ull;
      A.fl[2ll * r] = (unsigned long long)(h > 0) | ((unsigned long long)(l > 0) << 32);
      A.fl[2ll * r + 1] = 0ull;
    }
  }
}

__global__ void __launch_bounds__(kThreads) k_run_scatter(RunArgs A) {
  const int R = *A.cur.R;
  const int K = *A.Kp, Kn = *A.Knp;
  const long long S = (long long)A.m * K;
  auto eh = [&](long long r) { return (long long)(A.fl[2 * r] & 0xffffffffull); };
  auto el = [&](long long r) { return (long long)(A.fl[2 * r] >> 32); };
  const long long stride = (long long)gridDim.x * blockDim.x;
  const long long i0 = (long long)blockIdx.x * blockDim.x + threadIdx.x;
  if (i0 == 0) {
    const int tot = (int)(eh(R) + el(R));
    *A.nxt.R = tot;
    A.nxt.seg_run[(long long)A.m * Kn] = tot;
  }
  for (long long s = i0; s < S; s += stride) {  // next level's segment -> first run
    const int c = A.cidx[s % K];
    if (c < 0) continue;
    const long long chi = (s / K) * Kn + c;
    const long long r0 = A.cur.seg_run[s], r1 = A.cur.seg_run[s + 1];
    A.nxt.seg_run[chi] = (int32_t)(eh(r0) + el(r0));
    A.nxt.seg_run[chi + 1] = (int32_t)(eh(r1) + el(r0));
  }
  for (long long r = i0; r < R; r += stride) {
    const unsigned long long hl = A.run_hl[r];
    if (hl == 0ull) continue;
    const long long s = A.run_seg[r];
    const int c = A.cidx[s % K];
    const long long chi = (s / K) * Kn + c;
    const long long r0 = A.cur.seg_run[s], r1 = A.cur.seg_run[s + 1];
    const unsigned long long off = A.cnt[2 * r];  // exclusive (h, l) inside the parent segment
    const float v = A.cur.run_val[r];
    const unsigned h = (unsigned)(hl & 0xffffffffull), l = (unsigned)(hl >> 32);
    const int a = (int)(s / K);
    if (h) {
      const long long o = eh(r) + el(r0);
      const long long P = A.nxt.seg_start[chi] + (long long)(off & 0xffffffffull);
      A.nxt.run_val[o] = v;
      A.nxt.run_len[o] = (int32_t)h;
      A.nxt.run_pos[o] = P;
      fill_run_chunks(A.nxt.run_chunk, A.nxt, a, P, h, (int)o);
    }
    if (l) {
      const long long o = eh(r1) + el(r);
      const long long P = A.nxt.seg_start[chi + 1] + (long long)(off >> 32);
      A.nxt.run_val[o] = v;
      A.nxt.run_len[o] = (int32_t)l;
      A.nxt.run_pos[o] = P;
      fill_run_chunks(A.nxt.run_chunk, A.nxt, a, P, l, (int)o);
    }
  }
}

// ============================================================================ a4-a6 RLE: split on runs
// "the RLE elements are the candidates": with the values in runs and no missing values,
// split finding needs only each run's (G, H, count), a prefix over the runs of a segment and Eq. 2
// at every run end -- O(runs) work instead of a scan over every entry.
//   k_run_zero   clears the level's run records
//   k_run_agg    one warp per 256-entry chunk of the g-list: for every run touching the chunk, the
//                fp64 sums of g and h over the run's entries in the chunk (lane partials in item
//                order, then a butterfly, so a fixed association), added to the run's record as
//                exact 128-bit fixed point: every run total is exact and independent of the order
//                of the adds and of the attribute sharding (chunks are attribute-aligned)
//   k_run_split  one warp per (attribute, node) segment: exact prefix over its runs (32 runs per
//                step), the exact Eq. 2 gain at every run end but the segment's last (non-empty
//                low side), the segment's best (R12: largest gain, then the earlier run = the
//                larger value) posted as a node-best record
// segment of run r: the largest s with seg_run[s] <= r (runs are stored in segment order)
__device__ __forceinline__ long long run_segment(const int32_t* __restrict__ seg_run, long long S, int r) {
  long long lo = 0, hi = S - 1;
  while (lo < hi) {
    const long long mid = (lo + hi + 1) >> 1;
    if (seg_run[mid] <= r) lo = mid; else hi = mid - 1;
  }
  return lo;
}

// racc: per run a 5-word scan record: fixed-point g (lo, hi), h (lo, hi) -- cleared here, summed
// by k_run_agg -- and word 4 = run length | first run of its segment << 33 (the scan's reset flag)
__global__ void __launch_bounds__(kThreads) k_run_init(SplitArgs A, unsigned long long* __restrict__ racc) {
  const int K = *A.t.Kp;
  const int R = *A.t.tb.R;
  const long long S = (long long)A.t.m * K;
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < R; r += gridDim.x * blockDim.x) {
    const long long s = run_segment(A.t.tb.seg_run, S, r);
    unsigned long long* x = racc + 5ll * r;
    x[0] = 0ull; x[1] = 0ull; x[2] = 0ull; x[3] = 0ull;
    x[4] = (unsigned long long)(unsigned)A.t.tb.run_len[r] | ((unsigned long long)(A.t.tb.seg_run[s] == r) << 33);
  }
}

// k_run_agg: one warp per 256-entry chunk lying inside one run (nearly all chunks of
// low-cardinality lists), two chunks in flight per warp: lane sums in item order, a butterfly, one
// exact add per total.  Chunks holding several runs are listed (A.genlist) for k_run_agg_multi.
template <int HMODE>
#ifndef GBDT_RUNAGG_CTAS
#define GBDT_RUNAGG_CTAS 6  // C5 RLE split 2.42 -> 2.27 ms/tree
#endif
__global__ void __launch_bounds__(kThreads, GBDT_RUNAGG_CTAS) k_run_agg(SplitArgs A, unsigned long long* __restrict__ racc) {
  constexpr bool kH = HMODE == kHGather;
  __shared__ TabCache tc;
  const int lane = threadIdx.x & 31;
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0) return;
  tab_load(tc, A.t);
  __syncthreads();
  const Tables& tb = A.t.tb;
  const int Fg = A.fx[0], Fh = A.fx[1];
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < C; c += 2 * nw) {
    long long p0[2];
    int len[2], rb[2];
    bool one[2];
    double g[2][kItems];
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const int cu = c + u * nw;
      len[u] = 0;
      p0[u] = 0;
      rb[u] = 0;
      one[u] = false;
      if (cu < C) {
        const ChunkMeta M = chunk_meta(tc, A.t, K, cu);
        p0[u] = M.p0;
        len[u] = (int)(M.p1 - M.p0);
        rb[u] = tb.run_chunk[cu];
      }
      // the g loads do not wait for the run lookup (a multi-run chunk wastes them); full chunks
      // (nearly all) without per-item predicates
      const double* gp = A.glist + p0[u] + lane;
      if (len[u] == kChunk) {
#pragma unroll
        for (int k = 0; k < kItems; ++k) g[u][k] = __ldcs(gp + 32 * k);
      } else {
#pragma unroll
        for (int k = 0; k < kItems; ++k) g[u][k] = (32 * k + lane < len[u]) ? __ldcs(gp + 32 * k) : 0.0;
      }
    }
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const int cu = c + u * nw;
      if (cu < C) one[u] = tb.run_pos[rb[u]] + tb.run_len[rb[u]] >= p0[u] + len[u];
    }
#pragma unroll
    for (int u = 0; u < 2; ++u) {
      const int cu = c + u * nw;
      if (cu >= C) break;
      if (!one[u]) {
        if (lane == 0) A.genlist[atomicAdd(A.ngen, 1)] = cu;
        continue;
      }
      double sg = 0.0, sh = 0.0;
      if (len[u] == kChunk) {
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
          const double hk = kH ? __ldcs(A.hlist + p0[u] + 32 * k + lane) : hess_of<HMODE>(g[u][k]);
          sg = sg + g[u][k];
          sh = sh + hk;
        }
      } else {
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
          const bool in = 32 * k + lane < len[u];
          const double hk = in ? (kH ? __ldcs(A.hlist + p0[u] + 32 * k + lane) : hess_of<HMODE>(g[u][k])) : 0.0;
          sg = sg + g[u][k];
          sh = sh + hk;
        }
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) {
        sg = sg + __shfl_xor_sync(0xffffffffu, sg, o);
        sh = sh + __shfl_xor_sync(0xffffffffu, sh, o);
      }
      // g and h totals converted and added by two lanes at once
      if (lane < 2) fx_atomic_add(racc + 5ll * rb[u] + 2 * lane, to_fx(lane ? sh : sg, lane ? Fh : Fg));
    }
  }
}

// k_run_root: the root level of the split on runs, one warp per 256-entry chunk (lane l on entries
// 8l .. 8l+7): g (and h) gathered by instance into the g-list (once per tree, L2 evict-last), and
// the run totals of the single-run chunks as in k_run_agg; other chunks are listed for
// k_run_agg_multi, which reads the g-list written here.
template <int HMODE>
#ifndef GBDT_RUNROOT_CTAS
#define GBDT_RUNROOT_CTAS 0  // 0: the compiler's choice (a minimum of 1 CTA/SM would let it take more registers)
#endif
#if GBDT_RUNROOT_CTAS > 0
#define LB_GBDT_RUNROOT_CTAS __launch_bounds__(kThreads, GBDT_RUNROOT_CTAS)
#else
#define LB_GBDT_RUNROOT_CTAS __launch_bounds__(kThreads)
#endif
__global__ void LB_GBDT_RUNROOT_CTAS k_run_root(SplitArgs A, unsigned long long* __restrict__ racc) {
  constexpr bool kH = HMODE == kHGather;
  __shared__ TabCache tc;
  const int lane = threadIdx.x & 31;
  const int K = *A.t.Kp;
  const int C = *A.t.tb.C;
  if (K == 0) return;
  tab_load(tc, A.t);
  __syncthreads();
  const Tables& tb = A.t.tb;
  const int Fg = A.fx[0], Fh = A.fx[1];
  const unsigned long long pol_keep = policy_evict_last();
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int c = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; c < C; c += nw) {
    const ChunkMeta M = chunk_meta(tc, A.t, K, c);
    const long long p1 = M.p1;
    const long long base = M.p0 + (long long)lane * kItems;
    const int rb = tb.run_chunk[c];
    double g[kItems], h[kItems];
#pragma unroll
    for (int k = 0; k < kItems; ++k) { g[k] = 0.0; h[k] = 0.0; }
    if (base < p1) {
      const int4 i0 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base));
      const int4 i1 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base + 4));
      const int id[kItems] = {i0.x, i0.y, i0.z, i0.w, i1.x, i1.y, i1.z, i1.w};
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (base + k < p1) {
          g[k] = ld_keep(A.g + id[k], pol_keep);
          h[k] = kH ? ld_keep(A.h + id[k], pol_keep) : hess_of<HMODE>(g[k]);
        }
      }
      if (base + kItems <= p1) {  // lists are padded to 4 entries only: never write past the chunk
        double2* go = reinterpret_cast<double2*>(A.glist + base);
#pragma unroll
        for (int q = 0; q < kItems / 2; ++q) __stcs(go + q, make_double2(g[2 * q], g[2 * q + 1]));
        if (kH) {
          double2* ho = reinterpret_cast<double2*>(A.hlist + base);
#pragma unroll
          for (int q = 0; q < kItems / 2; ++q) __stcs(ho + q, make_double2(h[2 * q], h[2 * q + 1]));
        }
      } else {
#pragma unroll
        for (int k = 0; k < kItems; ++k)
          if (base + k < p1) {
            A.glist[base + k] = g[k];
            if (kH) A.hlist[base + k] = h[k];
          }
      }
    }
    if (tb.run_pos[rb] + tb.run_len[rb] < p1) {  // several runs: k_run_agg_multi
      if (lane == 0) A.genlist[atomicAdd(A.ngen, 1)] = c;
      continue;
    }
    double sg = ((g[0] + g[1]) + (g[2] + g[3])) + ((g[4] + g[5]) + (g[6] + g[7]));
    double sh = ((h[0] + h[1]) + (h[2] + h[3])) + ((h[4] + h[5]) + (h[6] + h[7]));
#pragma unroll
    for (int o = 16; o; o >>= 1) {
      sg = sg + __shfl_xor_sync(0xffffffffu, sg, o);
      sh = sh + __shfl_xor_sync(0xffffffffu, sh, o);
    }
    if (lane == 0) {
      fx_atomic_add(racc + 5ll * rb, to_fx(sg, Fg));
      fx_atomic_add(racc + 5ll * rb + 2, to_fx(sh, Fh));
    }
  }
}

// k_run_agg_multi: the listed chunks holding several runs, lane l on entries 8l .. 8l+7 (blocked).
// The runs starting inside the chunk mark a 256-bit head mask, a segmented scan (in-lane, then
// across the lanes) forms every run piece's sum at its last entry, and that lane adds it --
// O(entries) work whatever the number of runs.
template <int HMODE>
__global__ void __launch_bounds__(kThreads) k_run_agg_multi(SplitArgs A, unsigned long long* __restrict__ racc) {
  constexpr bool kH = HMODE == kHGather;
  __shared__ unsigned heads[kWarps][kChunk / 32];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const int K = *A.t.Kp;
  const int NL = *A.ngen;
  if (K == 0) return;
  const Tables& tb = A.t.tb;
  const int Fg = A.fx[0], Fh = A.fx[1];
  const int nw = (gridDim.x * blockDim.x) >> 5;
  unsigned* hw = heads[wid];
  for (int i = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; i < NL; i += nw) {
    const int c = A.genlist[i];
    const int a = tb.chunk_attr[c];
    const long long cs = tb.col_start[a], ce = cs + tb.col_len[a];
    const long long p0 = cs + (long long)(c - tb.chunk_start[a]) * kChunk;
    const int len = (int)(min(p0 + (long long)kChunk, ce) - p0);
    const int rb = tb.run_chunk[c];
    const int re = p0 + len < ce ? tb.run_chunk[c + 1] : tb.seg_run[(long long)a * K + K] - 1;
    const int q0 = kItems * lane;
    double g[kItems], h[kItems];
    if (q0 + kItems <= len) {
      const double2* gp = reinterpret_cast<const double2*>(A.glist + p0 + q0);
#pragma unroll
      for (int j = 0; j < kItems / 2; ++j) {
        const double2 z = __ldcs(gp + j);
        g[2 * j] = z.x;
        g[2 * j + 1] = z.y;
      }
      if (kH) {
        const double2* hp = reinterpret_cast<const double2*>(A.hlist + p0 + q0);
#pragma unroll
        for (int j = 0; j < kItems / 2; ++j) {
          const double2 z = __ldcs(hp + j);
          h[2 * j] = z.x;
          h[2 * j + 1] = z.y;
        }
      }
    } else {
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        g[k] = q0 + k < len ? __ldcs(A.glist + p0 + q0 + k) : 0.0;
        if (kH) h[k] = q0 + k < len ? __ldcs(A.hlist + p0 + q0 + k) : 0.0;
      }
    }
    if (!kH) {
#pragma unroll
      for (int k = 0; k < kItems; ++k) h[k] = q0 + k < len ? hess_of<HMODE>(g[k]) : 0.0;
    }
    // heads: the first entries of the runs that start inside the chunk (after its first entry)
    if (lane < kChunk / 32) hw[lane] = 0u;
    __syncwarp();
    for (int r = rb + 1 + lane; r <= re; r += 32) {
      const long long q = tb.run_pos[r] - p0;
      if (q > 0 && q < len) atomicOr(&hw[q >> 5], 1u << (q & 31));
    }
    __syncwarp();
    const unsigned hword = hw[lane >> 2];
    const unsigned hb = (hword >> ((lane & 3) * 8)) & 0xffu;  // heads among the lane's items
    // heads before the lane's first item (positions 1 .. q0-1): the run of its first item
    int before = 0;
#pragma unroll
    for (int wdx = 0; wdx < kChunk / 32; ++wdx)
      if (wdx < (lane >> 2)) before += __popc(hw[wdx]);
    before += __popc(hword & ((1u << ((lane & 3) * 8)) - 1u));
    // the head bit of the entry after the lane's last item
    const bool next_head = (q0 + kItems < kChunk) && ((hw[(q0 + kItems) >> 5] >> ((q0 + kItems) & 31)) & 1u);
    __syncwarp();  // hw is rewritten by the warp's next chunk
    double pg[kItems], ph[kItems];
    double rg = 0.0, rh = 0.0;
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if ((hb >> k) & 1u) { rg = 0.0; rh = 0.0; }
      rg = rg + g[k];
      rh = rh + h[k];
      pg[k] = rg;
      ph[k] = rh;
    }
    // segmented inclusive scan of the lane tails across the lanes (lane 0 starts the chunk)
    double ig = rg, ih = rh;
    int fl = (hb != 0u || lane == 0) ? 1 : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const double yg = __shfl_up_sync(0xffffffffu, ig, o), yh = __shfl_up_sync(0xffffffffu, ih, o);
      const int yf = __shfl_up_sync(0xffffffffu, fl, o);
      if (lane >= o) {
        if (!fl) { ig = yg + ig; ih = yh + ih; }
        fl |= yf;
      }
    }
    double cg = __shfl_up_sync(0xffffffffu, ig, 1), ch = __shfl_up_sync(0xffffffffu, ih, 1);
    if (lane == 0) { cg = 0.0; ch = 0.0; }
    int run = rb + before;
    bool open = true;  // the lane's current piece began in an earlier lane
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      const int q = q0 + k;
      if ((hb >> k) & 1u) { ++run; open = false; }
      const bool end = q < len && (q + 1 == len || (k + 1 < kItems ? ((hb >> (k + 1)) & 1u) != 0u : next_head));
      if (end) {
        const double tg = open ? cg + pg[k] : pg[k], th = open ? ch + ph[k] : ph[k];
        fx_atomic_add(racc + 5ll * run, to_fx(tg, Fg));
        fx_atomic_add(racc + 5ll * run + 2, to_fx(th, Fh));
      }
    }
  }
}

// One warp per 256 consecutive runs (8 steps of 32): the candidate at the end of run r (not the
// last run of its segment) has the high side = runs up to r, whose totals are the exact carry of
// run r+1 (k_scan3, converted once to fp64).  Segmented argmax over the lanes (segments are
// contiguous runs), the best of a segment piece carried across steps; a piece that ends its
// segment or the warp's range posts one record (<= runs/256 + segments records per level).
constexpr int kRunSteps = 8;
__global__ void __launch_bounds__(kThreads) k_run_split(SplitArgs A, const unsigned long long* __restrict__ rcar) {
  const int lane = threadIdx.x & 31;
  const int K = *A.t.Kp;
  if (K == 0) return;
  const Tables& tb = A.t.tb;
  const int R = *tb.R;
  const long long S = (long long)A.t.m * K;
  const int epoch = *A.epochp;
  const double lam = A.lam;
  const int nw = (gridDim.x * blockDim.x) >> 5;
  for (int base = ((blockIdx.x * blockDim.x + threadIdx.x) >> 5) * (32 * kRunSteps); base < R;
       base += nw * 32 * kRunSteps) {
    long long cs_ = -1;  // segment of the carried best (-1: none)
    unsigned long long ckey = 0ull;
    int cr = -1;
    for (int step = 0; step < kRunSteps; ++step) {
      const int rb = base + 32 * step;
      if (rb >= R) break;
      const int r = rb + lane;
      const bool act = r < R;
      long long s = act ? run_segment(tb.seg_run, S, r) : LLONG_MAX;
      const bool seg_last = act && r + 1 >= tb.seg_run[s + 1];
      const bool cand = act && !seg_last;
      unsigned long long key = 0ull;
      double GL = 0.0, HL = 0.0;
      int j = 0;
      if (act) j = (int)(s % K);
      if (cand) {
        const CarryD cx = carry_load(rcar + 5ll * (r + 1));
        GL = cx.g;
        HL = cx.h;
        key = gain_key(eq2_gain(GL, HL, A.nodes.G[j], A.nodes.H[j], lam, A.nodes.pterm[j]));
      }
      // segmented argmax over the lanes: larger key, then the earlier run (R12)
      unsigned long long bk = key;
      int bl = lane;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long yk = __shfl_up_sync(0xffffffffu, bk, o);
        const int yl = __shfl_up_sync(0xffffffffu, bl, o);
        const long long ys = __shfl_up_sync(0xffffffffu, s, o);
        if (lane >= o && ys == s && yk >= bk) { bk = yk; bl = yl; }
      }
      // the first piece of the step continues the carried segment
      if (s == cs_ && ckey >= bk && ckey) { bk = ckey; bl = -1 - cr; }  // encode a carried run as < 0
      const long long sn = __shfl_down_sync(0xffffffffu, s, 1);
      const bool piece_end = act && (lane == 31 || sn != s);
      const bool range_end = act && (lane == 31 ? step == kRunSteps - 1 : false) || (act && r == R - 1);
      // carry: the last lane's piece when it does not end its segment
      const unsigned long long lk = __shfl_sync(0xffffffffu, bk, 31);
      const int ll = __shfl_sync(0xffffffffu, bl, 31);
      const long long ls = __shfl_sync(0xffffffffu, s, 31);
      const bool lend = __shfl_sync(0xffffffffu, seg_last, 31);
      const int lr = ll < 0 ? -1 - ll : rb + ll;
      if (piece_end && (seg_last || range_end) && bk) {
        const int wr = bl < 0 ? -1 - bl : rb + bl;
        const CarryD cx = carry_load(rcar + 5ll * (wr + 1));
        const long long ws = bl < 0 ? cs_ : s;
        const int wj = (int)(ws % K);
        Rec rc;
        rc.GL = cx.g;
        rc.HL = cx.h;
        rc.cntL = cx.c;
        rc.gain = eq2_gain(cx.g, cx.h, A.nodes.G[wj], A.nodes.H[wj], lam, A.nodes.pterm[wj]);
        rc.value = tb.run_val[wr];
        rc.attr = A.t.a_base + (int)(ws / K);
        rc.dir = 0;
        rc.node = wj;
        rc.epoch = epoch;
        rc.shard = A.shard;
        rc.pos = tb.run_pos[wr] + tb.run_len[wr] - 1;
        post_global(A, rc);
      }
      if (ls != LLONG_MAX && !lend) { cs_ = ls; ckey = lk; cr = lr; } else { cs_ = -1; ckey = 0ull; cr = -1; }
    }
  }
}

// ---------------------------------------------------------------------------- RLE split ablation
// "Splitting RLE with decompression" (Fig. 6), the baseline the paper's direct RLE split
// (Fig. 7) is measured against: the level's runs are decompressed into the value
// list, the entries are partitioned as plain lists (values moving with them), and the children
// are compressed again -- one run per maximal group of equal values inside each (node, attribute)
// segment.  Produces exactly the tables of the direct split (RLE(filter(root column))).
__global__ void __launch_bounds__(kThreads) k_rle_decompress(Tables tb, float* __restrict__ val) {
  const int R = *tb.R;
  const int lane = threadIdx.x & 31;
  for (int r = blockIdx.x * kWarps + (threadIdx.x >> 5); r < R; r += gridDim.x * kWarps) {
    const long long P = tb.run_pos[r];
    const int L = tb.run_len[r];
    const float v = tb.run_val[r];
    for (int q = lane; q < L; q += 32) val[P + q] = v;
  }
}

// Encoding the next level's lists, entry-parallel (one warp per 256-entry chunk of the next
// level's tables): an entry starts a run iff it starts its (node, attribute) segment or its value
// differs from the previous entry's.  Segment starts are marked in a bitmap first.
__device__ __forceinline__ bool enc_head(const Tables& tn, const float* val, const uint32_t* sbits, long long p) {
  return ((sbits[p >> 5] >> (p & 31)) & 1u) || val[p] != val[p - 1];
}

__global__ void k_enc_mark(Tables tn, int m, const int32_t* __restrict__ Knp, uint32_t* __restrict__ sbits) {
  const long long S = (long long)m * *Knp;
  for (long long s = (long long)blockIdx.x * blockDim.x + threadIdx.x; s < S; s += (long long)gridDim.x * blockDim.x)
    if (tn.seg_cnt[s] > 0) {
      const long long p = tn.seg_start[s];
      atomicOr(sbits + (p >> 5), 1u << (p & 31));
    }
}

__device__ __forceinline__ void enc_chunk_range(const Tables& tn, int c, long long& p0, long long& p1, int& a) {
  a = tn.chunk_attr[c];
  const long long cs = tn.col_start[a];
  p0 = cs + (long long)(c - tn.chunk_start[a]) * kChunk;
  p1 = min(p0 + (long long)kChunk, cs + tn.col_len[a]);
}

__global__ void __launch_bounds__(kThreads) k_enc_count(Tables tn, const float* __restrict__ val,
                                                        const uint32_t* __restrict__ sbits, uint32_t* __restrict__ cnt) {
  const int C = *tn.C;
  const int lane = threadIdx.x & 31;
  for (int c = blockIdx.x * kWarps + (threadIdx.x >> 5); c <= C; c += gridDim.x * kWarps) {
    uint32_t k = 0;
    if (c < C) {
      long long p0, p1;
      int a;
      enc_chunk_range(tn, c, p0, p1, a);
      for (long long p = p0 + lane; p < p1; p += 32) k += enc_head(tn, val, sbits, p) ? 1u : 0u;
      for (int o = 16; o; o >>= 1) k += __shfl_xor_sync(0xffffffffu, k, o);
    }
    if (lane == 0) cnt[c] = k;
  }
}

// single-CTA exclusive scan of n counts in place; *total = the sum
__global__ void k_enc_scan(uint32_t* __restrict__ a, const int32_t* __restrict__ np, int32_t* __restrict__ total) {
  __shared__ uint32_t ws[32];
  __shared__ uint32_t carry;
  const long long n = (long long)*np + 1;
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  for (long long base = 0; base < n; base += blockDim.x) {
    const long long i = base + threadIdx.x;
    const uint32_t x = i < n ? a[i] : 0u;
    uint32_t incl = x;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += y;
    }
    if (lane == 31) ws[w] = incl;
    __syncthreads();
    if (w == 0) {
      const uint32_t s0 = lane < nw ? ws[lane] : 0u;
      uint32_t si = s0;
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, si, o);
        if (lane >= o) si += y;
      }
      if (lane < nw) ws[lane] = si - s0;
    }
    __syncthreads();
    const uint32_t c = carry;
    if (i < n) {
      a[i] = c + ws[w] + incl - x;
      if (i == n - 1) *total = (int32_t)(c + ws[w] + incl - x);
    }
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) carry = c + ws[w] + incl;
    __syncthreads();
  }
}

// run values / positions (heads ranked by ballots); a segment's first run recorded in seg_run
__global__ void __launch_bounds__(kThreads) k_enc_heads(Tables tn, int m, const int32_t* __restrict__ Knp,
                                                        const float* __restrict__ val, const uint32_t* __restrict__ sbits,
                                                        const uint32_t* __restrict__ base) {
  const int C = *tn.C, Kn = *Knp;
  const int lane = threadIdx.x & 31;
  for (int c = blockIdx.x * kWarps + (threadIdx.x >> 5); c < C; c += gridDim.x * kWarps) {
    long long p0, p1;
    int a;
    enc_chunk_range(tn, c, p0, p1, a);
    uint32_t r = base[c];
    for (long long q = p0; q < p1; q += 32) {
      const long long p = q + lane;
      const bool h = p < p1 && enc_head(tn, val, sbits, p);
      const unsigned hm = __ballot_sync(0xffffffffu, h);
      if (h) {
        const uint32_t rr = r + __popc(hm & ((1u << lane) - 1u));
        tn.run_val[rr] = val[p];
        tn.run_pos[rr] = p;
        if ((sbits[p >> 5] >> (p & 31)) & 1u) {  // a segment start: which segment of attribute a
          const int64_t* ss = tn.seg_start + (long long)a * Kn;
          int lo = 0, hi = Kn - 1;  // the non-empty segment starting at p: the last with start <= p
          while (lo < hi) {
            const int mid = (lo + hi + 1) >> 1;
            if (ss[mid] <= p) lo = mid; else hi = mid - 1;
          }
          tn.seg_run[(long long)a * Kn + lo] = (int32_t)rr;
        }
      }
      r += __popc(hm);
    }
  }
}

// run lengths (up to the next run or the segment's end) and the run -> chunk index
__global__ void __launch_bounds__(kThreads) k_enc_len(Tables tn, int m, const int32_t* __restrict__ Knp) {
  const int R = *tn.R, Kn = *Knp;
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < R; r += gridDim.x * blockDim.x) {
    const long long p = tn.run_pos[r];
    int lo = 0, hi = m - 1;  // attribute of p
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (tn.col_start[mid] <= p) lo = mid; else hi = mid - 1;
    }
    const int a = lo;
    const int64_t* ss = tn.seg_start + (long long)a * Kn;
    const int64_t* sc = tn.seg_cnt + (long long)a * Kn;
    int j0 = 0, j1 = Kn - 1;  // segment of p: the last with start <= p (segments tile the list)
    while (j0 < j1) {
      const int mid = (j0 + j1 + 1) >> 1;
      if (ss[mid] <= p) j0 = mid; else j1 = mid - 1;
    }
    const long long se = ss[j0] + sc[j0];
    const long long nx = r + 1 < R ? tn.run_pos[r + 1] : se;
    const long long L = min(nx, se) - p;
    tn.run_len[r] = (int32_t)L;
    fill_run_chunks(tn.run_chunk, tn, a, p, L, r);
  }
}

// empty segments point at the next segment's first run; seg_run[S] = R (one thread, backwards)
__global__ void k_enc_segfix(Tables tn, int m, const int32_t* __restrict__ Knp) {
  const long long S = (long long)m * *Knp;
  int next = *tn.R;
  tn.seg_run[S] = next;
  for (long long s = S - 1; s >= 0; --s) {
    if (tn.seg_cnt[s] == 0) tn.seg_run[s] = next;
    next = tn.seg_run[s];
  }
}

template <class KernelT>
unsigned grid_for(KernelT kern, size_t smem, int sms) {
  if (smem) GBDT_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  GBDT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kThreads, smem));
  if (occ < 1) fail(GBDT_E_CUDA, "kernel does not fit on an SM");
  return (unsigned)(occ * sms);
}


size_t fast_smem(int hmode) { return hmode == kHGather ? sizeof(FastSmem<true>) : sizeof(FastSmem<false>); }

template <int HM, bool kR>
void launch_fast(const SplitArgs& A, unsigned grid, cudaStream_t st) {
  k_sf_fast<HM, kR><<<grid, kThreads, fast_smem(HM), st>>>(A);
}
template <int HM, bool kM, bool kT, bool kR>
void launch_gen(const SplitArgs& A, unsigned grid, cudaStream_t st) {
  k_sf_gen<HM, kM, kT, kR><<<grid, kThreads, 0, st>>>(A);
}

template <int HM>
void launch_short(const SplitArgs& A, bool missing, bool rle, unsigned grid, cudaStream_t st) {
  if (missing) { if (rle) k_sf_short<HM, true, true><<<grid, kThreads, 0, st>>>(A); else k_sf_short<HM, true, false><<<grid, kThreads, 0, st>>>(A); }
  else { if (rle) k_sf_short<HM, false, true><<<grid, kThreads, 0, st>>>(A); else k_sf_short<HM, false, false><<<grid, kThreads, 0, st>>>(A); }
}

template <bool kFx>
void launch_scan(const int32_t* Cp, unsigned long long* in, unsigned long long* gbuf, unsigned long long* out,
                 unsigned groups, cudaStream_t st, const int32_t* fx = nullptr) {
  if (groups == 1) {  // one group (e.g. the plan's scan over the attributes): its carry is zero --
    // gbuf is never written when a buffer's bound is one group, and it starts zeroed
    k_scan3<kFx><<<1, kThreads, 0, st>>>(Cp, in, gbuf, out, fx);
    GBDT_LAUNCH_CHECK();
    count_launch(1);
    return;
  }
  k_scan1<kFx><<<groups, kThreads, 0, st>>>(Cp, in, gbuf);
  k_scan2<kFx><<<1, kScan2Threads, 0, st>>>(Cp, gbuf);
  k_scan3<kFx><<<groups, kThreads, 0, st>>>(Cp, in, gbuf, out, fx);
  GBDT_LAUNCH_CHECK();
  count_launch(3);
}

// Present totals of every segment (missing values): the partial written by k_chunk_agg at the
// segment's last entry, plus the exact carry of that chunk when the segment began before it.
__global__ void __launch_bounds__(kThreads) k_seg_totals(SplitArgs A) {
  const int K = *A.t.Kp;
  const long long S = (long long)A.t.m * K;
  const bool sp = A.t.sflag && K <= 32;  // the short path's segments sum their own totals
  const bool la = sp && A.longa;          // ... so only the other attributes' segments are walked
  const long long N = la ? (long long)A.nlong * K : S;
  for (long long t = blockIdx.x * (long long)blockDim.x + threadIdx.x; t < N; t += (long long)gridDim.x * blockDim.x) {
    const long long s = la ? (long long)A.longa[t / K] * K + t % K : t;
    if (A.t.tb.seg_cnt[s] == 0) continue;
    if (sp && !la && A.t.sflag[s / K]) continue;
    const int ce = A.segEnd[s];
    if (ce < 0) continue;
    const CarryD cx = carry_load(A.carry + 5ll * ce);
    A.segPG_out[s] = cx.g + A.segPG_out[s];
    A.segPH_out[s] = cx.h + A.segPH_out[s];
  }
}

}  // namespace

void LevelKernels::init(int device) {
  GBDT_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
  grid_fast[0][0] = grid_for(k_sf_fast<0, false>, fast_smem(0), sms);
  grid_fast[0][1] = grid_for(k_sf_fast<0, true>, fast_smem(0), sms);
  grid_fast[1][0] = grid_for(k_sf_fast<1, false>, fast_smem(1), sms);
  grid_fast[1][1] = grid_for(k_sf_fast<1, true>, fast_smem(1), sms);
  grid_fast[2][0] = grid_for(k_sf_fast<2, false>, fast_smem(2), sms);
  grid_fast[2][1] = grid_for(k_sf_fast<2, true>, fast_smem(2), sms);
  grid_gen = grid_for(k_sf_gen<2, true, false, true>, 0, sms);  // the largest variant
  grid_short = grid_for(k_sf_short<2, true, true>, 0, sms);
  grid_sl = grid_for(k_short_split<2, true>, 0, sms);
  grid_agg[0] = grid_for(k_chunk_agg<0, true>, 0, sms);
  grid_agg[1] = grid_for(k_chunk_agg<1, true>, 0, sms);
  grid_agg[2] = grid_for(k_chunk_agg<2, true>, 0, sms);
  grid_agg_list[0] = grid_for(k_chunk_agg<0, false>, 0, sms);
  grid_agg_list[1] = grid_for(k_chunk_agg<1, false>, 0, sms);
  grid_agg_list[2] = grid_for(k_chunk_agg<2, false>, 0, sms);
  grid_scatter[0][0] = grid_for(k_part_scatter<0, false, false>, 0, sms);
  grid_scatter[1][0] = grid_for(k_part_scatter<1, false, false>, 0, sms);
  grid_scatter[2][0] = grid_for(k_part_scatter<2, false, false>, 0, sms);
  grid_scatter[0][1] = grid_for(k_part_scatter<0, false, true>, 0, sms);
  grid_scatter[1][1] = grid_for(k_part_scatter<1, false, true>, 0, sms);
  grid_scatter[2][1] = grid_for(k_part_scatter<2, false, true>, 0, sms);
  grid_count = grid_for(k_part_count, 0, sms);
  grid_count_dense = grid_for(k_part_count_dense, 0, sms);
  fused_init(sms);
  grid_fused = std::max(fused_grid(0), fused_grid(1));
}

unsigned LevelKernels::scan_groups(int64_t max_chunks) {
  return (unsigned)std::max<int64_t>(1, (max_chunks + kScanGroup - 1) / kScanGroup);
}

void LevelKernels::tile_prefix(const SplitArgs& A, int hmode, bool gather, unsigned groups, cudaStream_t st) {
  if (gather) {
    if (hmode == 0) k_chunk_agg<0, true><<<grid_agg[0], kThreads, 0, st>>>(A);
    else if (hmode == 1) k_chunk_agg<1, true><<<grid_agg[1], kThreads, 0, st>>>(A);
    else k_chunk_agg<2, true><<<grid_agg[2], kThreads, 0, st>>>(A);
  } else {
    if (hmode == 0) k_chunk_agg<0, false><<<grid_agg_list[0], kThreads, 0, st>>>(A);
    else if (hmode == 1) k_chunk_agg<1, false><<<grid_agg_list[1], kThreads, 0, st>>>(A);
    else k_chunk_agg<2, false><<<grid_agg_list[2], kThreads, 0, st>>>(A);
  }
  GBDT_LAUNCH_CHECK();
  count_launch();
  launch_scan<true>(A.t.tb.C, A.cagg, A.sgrp, A.carry, groups, st, A.fx);
  if (A.segEnd) {
    k_seg_totals<<<(unsigned)(sms * 4), kThreads, 0, st>>>(A);
    GBDT_LAUNCH_CHECK();
    count_launch();
  }
}

void LevelKernels::split_find(const SplitArgs& A, int hmode, bool missing, bool rle, cudaStream_t st) {
  const unsigned gg = grid_gen;
#if GBDT_SF_SHORT_KERNEL
  // sparse lists (missing values): their short chunks go through k_sf_short; without missing
  // values the only short chunks are segment-crossing list tails, which k_sf_gen takes
  if (missing) {
    if (hmode == 0) launch_short<0>(A, missing, rle, grid_short, st);
    else if (hmode == 1) launch_short<1>(A, missing, rle, grid_short, st);
    else launch_short<2>(A, missing, rle, grid_short, st);
    GBDT_LAUNCH_CHECK();
    count_launch();
  }
#endif
  if (!missing) {  // single-segment chunks stream through k_sf_fast; the rest go through k_sf_gen
    const unsigned gf = grid_fast[hmode][rle];
    if (hmode == 0) { if (rle) launch_fast<0, true>(A, gf, st); else launch_fast<0, false>(A, gf, st); }
    else if (hmode == 1) { if (rle) launch_fast<1, true>(A, gf, st); else launch_fast<1, false>(A, gf, st); }
    else { if (rle) launch_fast<2, true>(A, gf, st); else launch_fast<2, false>(A, gf, st); }
    if (hmode == 0) { if (rle) launch_gen<0, false, false, true>(A, gg, st); else launch_gen<0, false, false, false>(A, gg, st); }
    else if (hmode == 1) { if (rle) launch_gen<1, false, false, true>(A, gg, st); else launch_gen<1, false, false, false>(A, gg, st); }
    else { if (rle) launch_gen<2, false, false, true>(A, gg, st); else launch_gen<2, false, false, false>(A, gg, st); }
    count_launch(2);
  } else {
    if (hmode == 0) { if (rle) launch_gen<0, true, false, true>(A, gg, st); else launch_gen<0, true, false, false>(A, gg, st); }
    else if (hmode == 1) { if (rle) launch_gen<1, true, false, true>(A, gg, st); else launch_gen<1, true, false, false>(A, gg, st); }
    else { if (rle) launch_gen<2, true, false, true>(A, gg, st); else launch_gen<2, true, false, false>(A, gg, st); }
    count_launch();
  }
  GBDT_LAUNCH_CHECK();
}

void LevelKernels::seg_totals(const SplitArgs& A, int hmode, cudaStream_t st) {
  if (hmode == 0) launch_gen<0, true, true, false>(A, grid_gen, st);
  else if (hmode == 1) launch_gen<1, true, true, false>(A, grid_gen, st);
  else launch_gen<2, true, true, false>(A, grid_gen, st);
  GBDT_LAUNCH_CHECK();
  count_launch();
}

void LevelKernels::partition_count(const PartArgs& A, const PlanArgs& P, bool counted, unsigned groups,
                                   cudaStream_t st, const ShortList* sl) {
  if (counted) k_part_count<<<grid_count, kThreads, 0, st>>>(A, 1);
  else k_part_count_dense<<<grid_count_dense, kThreads, 0, st>>>(A);
  GBDT_LAUNCH_CHECK();
  count_launch();
  if (sl && sl->nb && !sl->inplace) {  // (in-place lists have no segments to count)
    k_short_count<<<(unsigned)(sms * 8), kThreads, 0, st>>>(A, *sl);
    GBDT_LAUNCH_CHECK();
    count_launch();
  }
  launch_scan<false>(A.t.tb.C, A.ccnt, A.sgrp, A.cpre, groups, st);
  const unsigned pg = (unsigned)std::max(1, std::min((P.m + kWarps) / kWarps, sms * 8));  // a warp per attribute
  k_plan_attr<<<pg, kThreads, 0, st>>>(P);
  launch_scan<false>(P.mp1, P.el, P.egrp, P.el, P.egroups, st);
  k_plan_seg<<<pg, kThreads, 0, st>>>(P);
  k_chunk_attr<<<(unsigned)(sms * 8), kThreads, 0, st>>>(P);
  GBDT_LAUNCH_CHECK();
  count_launch(3);
}

template <int HM, bool kR>
void launch_scatter(const LevelKernels& L, const PartArgs& A, cudaStream_t st) {
  if (A.cagg_next) k_part_scatter<HM, kR, true><<<L.grid_scatter[HM][1], kThreads, 0, st>>>(A);
  else k_part_scatter<HM, kR, false><<<L.grid_scatter[HM][0], kThreads, 0, st>>>(A);
}

void LevelKernels::partition_scatter(const PartArgs& A, int hmode, const RunArgs* rle, cudaStream_t st,
                                     const ShortList* sl) {
  if (sl && sl->nb && sl->inplace) {
    k_short_update<<<(unsigned)(sms * 8), kThreads, 0, st>>>(A, *sl);
    GBDT_LAUNCH_CHECK();
    count_launch();
  } else if (sl && sl->nb) {
    if (hmode == 0) k_short_scatter<0><<<(unsigned)(sms * 8), kThreads, 0, st>>>(A, *sl);
    else if (hmode == 1) k_short_scatter<1><<<(unsigned)(sms * 8), kThreads, 0, st>>>(A, *sl);
    else k_short_scatter<2><<<(unsigned)(sms * 8), kThreads, 0, st>>>(A, *sl);
    GBDT_LAUNCH_CHECK();
    count_launch();
  }
  if (rle) {
    if (hmode == 0) launch_scatter<0, true>(*this, A, st);
    else if (hmode == 1) launch_scatter<1, true>(*this, A, st);
    else launch_scatter<2, true>(*this, A, st);
    GBDT_LAUNCH_CHECK();
    k_run_count<<<(unsigned)(sms * 8), kThreads, 0, st>>>(*rle);
    GBDT_LAUNCH_CHECK();
    count_launch();
    launch_scan<false>(rle->cur.R, rle->cnt, rle->sgrp, rle->cnt, rle->groups, st);
    launch_scan<false>(rle->Rp1, rle->fl, rle->sgrp, rle->fl, rle->groups, st);
    k_run_scatter<<<(unsigned)(sms * 8), kThreads, 0, st>>>(*rle);
    count_launch();
  } else {
    if (hmode == 0) launch_scatter<0, false>(*this, A, st);
    else if (hmode == 1) launch_scatter<1, false>(*this, A, st);
    else launch_scatter<2, false>(*this, A, st);
  }
  GBDT_LAUNCH_CHECK();
  count_launch();
}

void LevelKernels::short_split(const SplitArgs& A, const ShortList& S, int hmode, bool gather, cudaStream_t st) {
  if (!S.nb) return;
  const unsigned g = grid_sl;
  if (gather) {
    if (hmode == 0) k_short_split<0, true><<<g, kThreads, 0, st>>>(A, S);
    else if (hmode == 1) k_short_split<1, true><<<g, kThreads, 0, st>>>(A, S);
    else k_short_split<2, true><<<g, kThreads, 0, st>>>(A, S);
  } else {
    if (hmode == 0) k_short_split<0, false><<<g, kThreads, 0, st>>>(A, S);
    else if (hmode == 1) k_short_split<1, false><<<g, kThreads, 0, st>>>(A, S);
    else k_short_split<2, false><<<g, kThreads, 0, st>>>(A, S);
  }
  GBDT_LAUNCH_CHECK();
  count_launch();
}

void LevelKernels::rle_decompress(const Tables& tb, float* val, cudaStream_t st) {
  k_rle_decompress<<<(unsigned)(sms * 8), kThreads, 0, st>>>(tb, val);
  GBDT_LAUNCH_CHECK();
  count_launch();
}

void LevelKernels::rle_encode(const Tables& tn, int m, const int32_t* Knp, const float* val, uint32_t* cnt,
                              uint32_t* sbits, size_t sbits_bytes, cudaStream_t st) {
  GBDT_CUDA(cudaMemsetAsync(sbits, 0, sbits_bytes, st));
  k_enc_mark<<<(unsigned)(sms * 4), kThreads, 0, st>>>(tn, m, Knp, sbits);
  k_enc_count<<<(unsigned)(sms * 8), kThreads, 0, st>>>(tn, val, sbits, cnt);
  k_enc_scan<<<1, 1024, 0, st>>>(cnt, tn.C, tn.R);
  k_enc_heads<<<(unsigned)(sms * 8), kThreads, 0, st>>>(tn, m, Knp, val, sbits, cnt);
  k_enc_len<<<(unsigned)(sms * 8), kThreads, 0, st>>>(tn, m, Knp);
  k_enc_segfix<<<1, 1, 0, st>>>(tn, m, Knp);
  GBDT_LAUNCH_CHECK();
  count_launch(6);
}

void LevelKernels::run_split(const SplitArgs& A, int hmode, bool root, unsigned long long* racc,
                             unsigned long long* rcar, unsigned long long* rsg, unsigned groups, cudaStream_t st) {
  k_run_init<<<(unsigned)(sms * 4), kThreads, 0, st>>>(A, racc);
  const unsigned ga = (unsigned)(sms * 8);
  if (root) {  // the g-list is gathered here
    if (hmode == 0) k_run_root<0><<<ga, kThreads, 0, st>>>(A, racc);
    else if (hmode == 1) k_run_root<1><<<ga, kThreads, 0, st>>>(A, racc);
    else k_run_root<2><<<ga, kThreads, 0, st>>>(A, racc);
  } else {
    if (hmode == 0) k_run_agg<0><<<ga, kThreads, 0, st>>>(A, racc);
    else if (hmode == 1) k_run_agg<1><<<ga, kThreads, 0, st>>>(A, racc);
    else k_run_agg<2><<<ga, kThreads, 0, st>>>(A, racc);
  }
  if (hmode == 0) k_run_agg_multi<0><<<ga, kThreads, 0, st>>>(A, racc);
  else if (hmode == 1) k_run_agg_multi<1><<<ga, kThreads, 0, st>>>(A, racc);
  else k_run_agg_multi<2><<<ga, kThreads, 0, st>>>(A, racc);
  GBDT_LAUNCH_CHECK();
  count_launch(3);
  launch_scan<true>(A.t.tb.R, racc, rsg, rcar, groups, st, A.fx);
  k_run_split<<<(unsigned)(sms * 4), kThreads, 0, st>>>(A, rcar);
  GBDT_LAUNCH_CHECK();
  count_launch();
}

void LevelKernels::chunk_desc(const SplitArgs& A, unsigned groups, cudaStream_t st) {
  k_desc<<<(unsigned)(sms * 8), kThreads, 0, st>>>(A);
  GBDT_LAUNCH_CHECK();
  count_launch();
  launch_scan<true>(A.t.tb.C, A.cagg, A.sgrp, A.carry, groups, st, A.fx);
}

}  // namespace gbdt
