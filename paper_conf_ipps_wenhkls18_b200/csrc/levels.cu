// levels.cu -- the per-level streaming kernels of the hot path on sm_100a:
//
//   k_sf          a3-a6: segmented prefix sum of (g, h, count) over every (node, attribute)
//                 segment of the level's attribute-sorted lists (Fig. 1), Eq. 2 gain at
//                 the end of every run of equal values, both missing directions
//                 (P:116), best split per node
//   k_part_*      a8: order-preserving stable partition of every segment into its two children,
//                 entries of new leaves dropped
//
// The work unit is a tile: 2048 consecutive entries of one attribute list (tiles never straddle
// attributes).  The segmented scan is done reduce-then-scan, so no CTA ever waits on another:
//   k_tile_agg   per tile: gathers g (h) of the tile's instances -- the only random access of the
//                level, into an L2-resident array (n x 8 B: 88 MB for the 11M-row config, loaded
//                evict-last) -- writes them as a contiguous g-list next to the attribute list, and
//                publishes the tile's segmented aggregate
//   k_tile_scan  one warp per attribute: exact segmented carry of every tile
//   k_sf         persistent, 3-stage shared-memory ring fed by TMA 1-D bulk copies
//                (cp.async.bulk / UBLKCP, mbarrier completion, evict-first) of the tile's value
//                list and g-list; computes in-tile prefixes + carry, the Eq. 2 gains and the
//                per-node argmax while the next two tiles stream in
//   k_part_count / k_part_tscan / k_part_plan / k_part_scatter   same count -> scan -> scatter
//                shape for the partition
//
// Determinism: inside a tile every sum has a fixed association.  Across tiles, each tile's fp64
// aggregate is converted ONCE to an exact 128-bit fixed-point integer (trunc(x * 2^F), F per tree),
// and the carry into a tile is the integer sum of its predecessors' published values, assembled by
// a CTA-wide decoupled look-back.  Integer addition is exact and associative, so the carry -- and
// every prefix, gain and tree built from it -- is bit-identical whatever the timing, the tile
// schedule, or the attribute sharding (tiles are attribute-aligned).  The partition's carry is an
// integer count and equally exact.
#include <algorithm>
#include <climits>

#include "kernels.cuh"

namespace gbdt {
namespace {

constexpr int kStages = 3;
constexpr int kSegCache = 32;     // segment starts/counts of a tile's attribute cached per stage
constexpr int kCtaK = 64;         // per-CTA node-best table when K <= kCtaK
constexpr int kTabCache = 64;     // attribute tables cached in smem when m <= kTabCache
constexpr int kPieceList = 32;
constexpr int kLiteBlocks = 4;    // target CTAs/SM of the light streaming kernels

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
__device__ __forceinline__ SVf shfl_idx(const SVf& x, int l) {
  return SVf{__shfl_sync(0xffffffffu, x.g, l), __shfl_sync(0xffffffffu, x.h, l),
             __shfl_sync(0xffffffffu, x.c, l), __shfl_sync(0xffffffffu, x.f, l)};
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
  return AM{__shfl_up_sync(0xffffffffu, x.gain, o), __shfl_up_sync(0xffffffffu, x.value, o),
            __shfl_up_sync(0xffffffffu, x.meta, o), __shfl_up_sync(0xffffffffu, x.f, o)};
}

// ============================================================================ tile plumbing
struct TabCache {
  int use;
  int tile_start[kTabCache + 1];
  long long col_start[kTabCache + 1];
  long long col_len[kTabCache];
};

__device__ __forceinline__ void tab_load(TabCache& tc, const TileArgs& A) {
  const bool use = A.m <= kTabCache;
  if (threadIdx.x == 0) tc.use = use;
  if (use) {
    for (int i = threadIdx.x; i <= A.m; i += blockDim.x) {
      tc.tile_start[i] = A.tb.tile_start[i];
      tc.col_start[i] = A.tb.col_start[i];
      if (i < A.m) tc.col_len[i] = A.tb.col_len[i];
    }
  }
}


// Tile metadata computed by one thread.
struct TileMeta {
  long long p0, p1, colend, sb;
  int t, a, u, pad;
};

__device__ __forceinline__ void tile_meta(const TabCache& tc, const TileArgs& A, int K, int t, TileMeta& M) {
  const bool c = tc.use;
  const int* ts = c ? tc.tile_start : A.tb.tile_start;
  int lo = 0, hi = A.m - 1;  // largest a with tile_start[a] <= t
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (ts[mid] <= t) lo = mid; else hi = mid - 1;
  }
  const int a = lo;
  const long long cs = c ? tc.col_start[a] : A.tb.col_start[a];
  const long long cl = c ? tc.col_len[a] : A.tb.col_len[a];
  M.t = t;
  M.a = a;
  M.u = t - ts[a];
  M.colend = cs + cl;
  M.p0 = cs + (long long)M.u * kTile;
  M.p1 = min(M.p0 + (long long)kTile, M.colend);
  M.sb = (long long)a * K;
}

// Segment (node) of each of the thread's items; head / piece-end / run-end masks.
template <bool kNeedVal>
__device__ __forceinline__ void assign_segments(const long long* ss, const long long* sc, long long p1, int K, long long base,
                                                unsigned vm, const float* v, float vnext, int* sj,
                                                unsigned& hm, unsigned& pem, unsigned& rem) {
  hm = pem = rem = 0;
  if (!vm) return;
  int lo = 0, hi = K - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
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
    if (seg_last || p + 1 == p1) pem |= 1u << k;
    if (kNeedVal) {
      const float nv = (k < kItems - 1) ? v[k + 1] : vnext;
      if (seg_last || nv != v[k]) rem |= 1u << k;
    } else if (seg_last) {
      rem |= 1u << k;
    }
  }
}

// ---- exact 128-bit fixed point: x -> trunc(x * 2^F).  F is chosen per tree so that every sum of
// |g| (|h|) over the level fits below 2^125; conversion of a given double is a pure function, and
// integer addition is associative, so cross-tile carries are bit-identical in any order.
__device__ __forceinline__ __int128 to_fx(double x, int F) {
  if (x == 0.0) return 0;
  const long long b = __double_as_longlong(x);
  const int e = (int)((b >> 52) & 0x7ff);
  const unsigned long long mant = (unsigned long long)(b & 0xfffffffffffffll) | (e ? (1ull << 52) : 0ull);
  const int sh = (e ? e : 1) - 1075 + F;
  unsigned __int128 v;
  if (sh >= 0) v = (unsigned __int128)mant << (sh > 74 ? 74 : sh);
  else v = (sh > -64) ? (unsigned __int128)(mant >> (-sh)) : (unsigned __int128)0;
  return b < 0 ? -(__int128)v : (__int128)v;
}
__device__ __forceinline__ double from_fx(__int128 v, int F) {
  const bool neg = v < 0;
  const unsigned __int128 u = neg ? (unsigned __int128)(-v) : (unsigned __int128)v;
  const double hi = (double)(unsigned long long)(u >> 64), lo = (double)(unsigned long long)u;
  double r = __dadd_rn(__dmul_rn(hi, 18446744073709551616.0), lo);
  r = __dmul_rn(r, __longlong_as_double((long long)(1023 - F) << 52));  // exact power of two
  return neg ? -r : r;
}
__device__ __forceinline__ __int128 shfl_xor128(__int128 v, int o) {
  const unsigned long long lo = __shfl_xor_sync(0xffffffffu, (unsigned long long)v, o);
  const unsigned long long hi = __shfl_xor_sync(0xffffffffu, (unsigned long long)((unsigned __int128)v >> 64), o);
  return (__int128)(((unsigned __int128)hi << 64) | lo);
}
__device__ __forceinline__ __int128 ld128(const unsigned long long* p) {
  return (__int128)(((unsigned __int128)__ldcg(p + 1) << 64) | __ldcg(p));
}
__device__ __forceinline__ void st128(unsigned long long* p, __int128 v) {
  p[0] = (unsigned long long)v;
  p[1] = (unsigned long long)((unsigned __int128)v >> 64);
}

struct FX {
  __int128 g, h;
  int c, f;
};

__device__ __forceinline__ void fx_publish(unsigned long long* dst, const FX& x) {
  st128(dst, x.g);
  st128(dst + 2, x.h);
  dst[4] = (unsigned long long)(unsigned)x.c | ((unsigned long long)(unsigned)x.f << 32);
}


struct FXV {
  __int128 g, h;
  int c, f;
};
__device__ __forceinline__ FXV fxv_comb(const FXV& l, const FXV& r) {  // segmented, exact
  if (r.f) return r;
  return FXV{l.g + r.g, l.h + r.h, l.c + r.c, l.f};
}
__device__ __forceinline__ __int128 shfl_up128(__int128 v, int o) {
  const unsigned long long lo = __shfl_up_sync(0xffffffffu, (unsigned long long)v, o);
  const unsigned long long hi = __shfl_up_sync(0xffffffffu, (unsigned long long)((unsigned __int128)v >> 64), o);
  return (__int128)(((unsigned __int128)hi << 64) | lo);
}
__device__ __forceinline__ void fxv_store(unsigned long long* dst, const FXV& x) {
  st128(dst, x.g);
  st128(dst + 2, x.h);
  dst[4] = (unsigned long long)(unsigned)x.c | ((unsigned long long)(unsigned)x.f << 32);
}
__device__ __forceinline__ FXV fxv_load(const unsigned long long* src) {
  const unsigned long long cf = src[4];
  return FXV{(__int128)(((unsigned __int128)src[1] << 64) | src[0]),
             (__int128)(((unsigned __int128)src[3] << 64) | src[2]), (int)(unsigned)cf, (int)(cf >> 32)};
}

template <int HMODE>
__device__ __forceinline__ double hess_of(double g) {
  if (HMODE == kHConst2) return 2.0;
  // logistic, 0/1 labels: y = [g < 0] (g = p - y with p in [0,1]); q = g + y; reading R5b
  const double q = g < 0.0 ? __dadd_rn(g, 1.0) : g;
  const double hh = __dmul_rn(q, __dsub_rn(1.0, q));
  return hh > 1e-16 ? hh : 1e-16;
}

// ============================================================================ a4: tile aggregates
// Per tile: gather g (h) of its instances (L2-resident, evict-last), write them as the tile's
// g-list (h-list), and publish the tile's segmented aggregate (sum since its last segment head,
// fixed in-tile association) as an exact fixed-point value.
template <int HMODE>
__global__ void __launch_bounds__(kThreads, kLiteBlocks) k_tile_agg(SplitArgs A) {
  __shared__ TabCache tc;
  __shared__ TileMeta sm;
  __shared__ SVf wtot[kWarps];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int K = *A.t.Kp;
  const int T = *A.t.tb.T;
  if (K == 0 || T == 0) return;
  const int Fg = A.fx[0], Fh = A.fx[1];
  tab_load(tc, A.t);
  __syncthreads();
  for (int t = blockIdx.x; t < T; t += gridDim.x) {
    if (tid == 0) tile_meta(tc, A.t, K, t, sm);
    __syncthreads();
    const long long p1 = sm.p1;
    const long long base = sm.p0 + (long long)tid * kItems;
    unsigned vm = 0;
    double g[kItems], h[kItems];
    if (base < p1) {
      const int4 i0 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base));
      const int4 i1 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base + 4));
      const int id[kItems] = {i0.x, i0.y, i0.z, i0.w, i1.x, i1.y, i1.z, i1.w};
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (base + k < p1) {
          vm |= 1u << k;
          g[k] = __ldg(A.g + id[k]);
          h[k] = HMODE == kHGather ? __ldg(A.h + id[k]) : hess_of<HMODE>(g[k]);
        } else {
          g[k] = 0.0; h[k] = 0.0;
        }
      }
      // lists are padded to 4 entries only: never write past the tile's own entries
      if (base + kItems <= p1) {
        double2* go = reinterpret_cast<double2*>(A.glist + base);
#pragma unroll
        for (int k = 0; k < kItems / 2; ++k) go[k] = make_double2(g[2 * k], g[2 * k + 1]);
        if (HMODE == kHGather) {
          double2* ho = reinterpret_cast<double2*>(A.hlist + base);
#pragma unroll
          for (int k = 0; k < kItems / 2; ++k) ho[k] = make_double2(h[2 * k], h[2 * k + 1]);
        }
      } else {
#pragma unroll
        for (int k = 0; k < kItems; ++k) {
          if (base + k < p1) {
            A.glist[base + k] = g[k];
            if (HMODE == kHGather) A.hlist[base + k] = h[k];
          }
        }
      }
    }
    int sj[kItems];
    unsigned hm, pem, rem;
    float vdummy[kItems];
    assign_segments<false>((const long long*)(A.t.tb.seg_start + sm.sb), (const long long*)(A.t.tb.seg_cnt + sm.sb),
                           p1, K, base, vm, vdummy, 0.f, sj, hm, pem, rem);
    SVf run = svf_zero();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1)) continue;
      if ((hm >> k) & 1) { run.g = g[k]; run.h = h[k]; run.c = 1; run.f = 1; }
      else { run.g = run.g + g[k]; run.h = run.h + h[k]; run.c += 1; }
    }
    SVf inc = run;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const SVf y = shfl_up(inc, o);
      if (lane >= o) inc = comb(y, inc);
    }
    if (lane == 31) wtot[wid] = inc;
    __syncthreads();
    if (tid == 0) {
      SVf agg = svf_zero();
      for (int w = 0; w < kWarps; ++w) agg = comb(agg, wtot[w]);
      fxv_store(A.tagg + 5ll * t, FXV{to_fx(agg.g, Fg), to_fx(agg.h, Fh), agg.c, agg.f});
    }
    __syncthreads();
  }
}

// One warp per attribute: exact segmented exclusive scan of the tile aggregates -> carry per tile.
__global__ void __launch_bounds__(256) k_tile_scan(SplitArgs A) {
  const int K = *A.t.Kp;
  if (K == 0) return;
  const int lane = threadIdx.x & 31;
  const int warps = gridDim.x * (blockDim.x >> 5);
  for (int a = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); a < A.t.m; a += warps) {
    const int t0 = A.t.tb.tile_start[a], t1 = A.t.tb.tile_start[a + 1];
    FXV carry{0, 0, 0, 0};
    for (int base = t0; base < t1; base += 32) {
      const int t = base + lane;
      FXV x{0, 0, 0, 0};
      if (t < t1) x = fxv_load(A.tagg + 5ll * t);
      FXV inc = x;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        FXV y;
        y.g = shfl_up128(inc.g, o);
        y.h = shfl_up128(inc.h, o);
        y.c = __shfl_up_sync(0xffffffffu, inc.c, o);
        y.f = __shfl_up_sync(0xffffffffu, inc.f, o);
        if (lane >= o) inc = fxv_comb(y, inc);
      }
      FXV exc;
      exc.g = shfl_up128(inc.g, 1);
      exc.h = shfl_up128(inc.h, 1);
      exc.c = __shfl_up_sync(0xffffffffu, inc.c, 1);
      exc.f = __shfl_up_sync(0xffffffffu, inc.f, 1);
      if (lane == 0) exc = FXV{0, 0, 0, 0};
      const FXV ex = fxv_comb(carry, exc);
      if (t < t1) fxv_store(A.carry + 5ll * t, ex);
      FXV last;
      {
        const unsigned long long lo = __shfl_sync(0xffffffffu, (unsigned long long)inc.g, 31);
        const unsigned long long hi = __shfl_sync(0xffffffffu, (unsigned long long)((unsigned __int128)inc.g >> 64), 31);
        last.g = (__int128)(((unsigned __int128)hi << 64) | lo);
        const unsigned long long lo2 = __shfl_sync(0xffffffffu, (unsigned long long)inc.h, 31);
        const unsigned long long hi2 = __shfl_sync(0xffffffffu, (unsigned long long)((unsigned __int128)inc.h >> 64), 31);
        last.h = (__int128)(((unsigned __int128)hi2 << 64) | lo2);
        last.c = __shfl_sync(0xffffffffu, inc.c, 31);
        last.f = __shfl_sync(0xffffffffu, inc.f, 31);
      }
      carry = fxv_comb(carry, last);
    }
  }
}

// ============================================================================ a3-a6: split find
struct StageMeta {
  long long p0, p1, colend, sb;
  int t, a, u, seg_cached;
  unsigned long long carry[5];
  long long seg_s[kSegCache];
  long long seg_c[kSegCache];
};

// lane 0 of warp 0: metadata of tile t and the TMA bulk loads of its lists into a stage; lanes
// fetch the tile's carry and the attribute's segment table with cp.async.
template <bool kVal, bool kH>
__device__ __forceinline__ void issue_stage(int lane, int t, int T, int K, const TabCache& tc,
                                            const SplitArgs& A, StageMeta& M, float* sval, double* sg,
                                            double* sh, unsigned long long* bar, unsigned long long pol) {
  if (lane == 0) {
    TileMeta tm;
    tm.t = t;
    M.t = t;
    if (t < T) {
      tile_meta(tc, A.t, K, t, tm);
      M.a = tm.a; M.u = tm.u; M.p0 = tm.p0; M.p1 = tm.p1; M.colend = tm.colend; M.sb = tm.sb;
      M.seg_cached = K <= kSegCache;
      const long long cs = tc.use ? tc.col_start[tm.a] : A.t.tb.col_start[tm.a];
      const long long cl = tc.use ? tc.col_len[tm.a] : A.t.tb.col_len[tm.a];
      const long long r1 = min((tm.p1 + 3) & ~3ll, cs + ((cl + 3) & ~3ll));  // 16-byte granules
      const uint32_t n = (uint32_t)(r1 - tm.p0);
      fence_proxy_async();
      mbar_arrive_expect_tx(bar, (kVal ? 4u * n : 0u) + 8u * n + (kH ? 8u * n : 0u));
      if (kVal) tma_load_1d(sval, A.t.val + tm.p0, 4u * n, bar, pol);
      tma_load_1d(sg, A.glist + tm.p0, 8u * n, bar, pol);
      if (kH) tma_load_1d(sh, A.hlist + tm.p0, 8u * n, bar, pol);
    }
  }
  __syncwarp();
  if (t < T) {
    if (lane < 5) cp_async8(&M.carry[lane], A.carry + 5ll * t + lane, pol);
    if (K <= kSegCache) {
      const long long sb = M.sb;
      for (int j = lane; j < K; j += 32) {
        cp_async8(&M.seg_s[j], A.t.tb.seg_start + sb + j, pol);
        cp_async8(&M.seg_c[j], A.t.tb.seg_cnt + sb + j, pol);
      }
    }
  }
}

struct SFSmem {
  float val[kStages][kTile];
  double g[kStages][kTile];
  StageMeta meta[kStages];
  unsigned long long bar[kStages];
  int npw;
  SVf wtot[kWarps], wcar[kWarps];
  AM mtot[kWarps], mcar[kWarps];
  unsigned char win[kTile];
  unsigned long long cg[kCtaK], ct[kCtaK];
  Rec cb[kCtaK];
  Rec pw[kPieceList];
  TabCache tc;
};

__device__ __forceinline__ void cta_merge(SFSmem& S) {
  const int n = min(S.npw, kPieceList);
  for (int q = 0; q < n; ++q) {
    const Rec& r = S.pw[q];
    const unsigned long long gk = gain_key(r.gain), tk = tie_key(r.attr, r.value, r.dir);
    const int j = r.node;
    if (gk > S.cg[j] || (gk == S.cg[j] && tk < S.ct[j])) { S.cg[j] = gk; S.ct[j] = tk; S.cb[j] = r; }
  }
  S.npw = 0;
}

template <int HMODE, bool kMissing, bool kTotals>
__global__ void __launch_bounds__(kThreads, 2) k_sf(SplitArgs A) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  SFSmem& S = *reinterpret_cast<SFSmem*>(smem_raw);
  double* sH = reinterpret_cast<double*>(smem_raw + ((sizeof(SFSmem) + 127) & ~size_t(127)));  // mode 2
  constexpr bool kH = HMODE == kHGather;

  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int K = *A.t.Kp;
  const int T = *A.t.tb.T;
  if (K == 0 || T == 0) return;
  const int epoch = *A.epochp;
  const int Fg = A.fx[0], Fh = A.fx[1];
  const bool cta_table = !kTotals && K <= kCtaK;
  const unsigned long long pol_stream = policy_evict_first();
  // static round-robin tiles (no inter-CTA dependencies: carries come from k_tile_scan)
  auto tile_of = [&](int i) { return (int)blockIdx.x + i * (int)gridDim.x; };
  if (tid == 0) {
    for (int s = 0; s < kStages; ++s) mbar_init(&S.bar[s], 1);
    fence_mbar_init();
    S.npw = 0;
  }
  tab_load(S.tc, A.t);
  for (int i = tid; i < kTile; i += kThreads) S.win[i] = 0;
  for (int j = tid; j < kCtaK; j += kThreads) { S.cg[j] = 0ull; S.ct[j] = ~0ull; }
  __syncthreads();
  auto issue = [&](int i) {
    const int s = i % kStages;
    if (wid == 0)
      issue_stage<!kTotals, kH>(lane, tile_of(i), T, K, S.tc, A, S.meta[s], S.val[s], S.g[s],
                                kH ? sH + (size_t)s * kTile : nullptr, &S.bar[s], pol_stream);
    cp_async_commit();
  };
  issue(0);
  issue(1);

  for (int it = 0;; ++it) {
    const int s0 = it % kStages;
    issue(it + 2);
    cp_async_wait<2>();                   // this tile's carry / segment table (cp.async)
    __syncthreads();
    if (tid == 0 && S.npw) cta_merge(S);
    const StageMeta& M = S.meta[s0];
    const int t = M.t;
    if (t >= T) break;
    mbar_wait(&S.bar[s0], (uint32_t)((it / kStages) & 1));  // this tile's lists (TMA)

    const long long p0 = M.p0, p1 = M.p1;
    const int ibase = tid * kItems;
    const long long base = p0 + ibase;
    // ---------------------------------------------------------------- items from shared memory
    float v[kItems];
    double g[kItems], h[kItems];
    int c[kItems];
    unsigned vm = 0;
    float vnext = 0.f;
#pragma unroll
    for (int k = 0; k < kItems; ++k)
      if (base + k < p1) vm |= 1u << k;
    if (!kTotals) {
      const float4 v0 = *reinterpret_cast<const float4*>(&S.val[s0][ibase]);
      const float4 v1 = *reinterpret_cast<const float4*>(&S.val[s0][ibase + 4]);
      v[0] = v0.x; v[1] = v0.y; v[2] = v0.z; v[3] = v0.w;
      v[4] = v1.x; v[5] = v1.y; v[6] = v1.z; v[7] = v1.w;
      if (base + kItems < p1) vnext = S.val[s0][ibase + kItems];
      else if (base + kItems < M.colend && base + kItems == p1) vnext = __ldg(A.t.val + p1);
    } else {
#pragma unroll
      for (int k = 0; k < kItems; ++k) v[k] = 0.f;
    }
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if ((vm >> k) & 1) {
        g[k] = S.g[s0][ibase + k];
        h[k] = kH ? sH[(size_t)s0 * kTile + ibase + k] : hess_of<HMODE>(g[k]);
      } else {
        g[k] = 0.0; h[k] = 0.0;
      }
    }
    int sj[kItems];
    unsigned hm, pem, rem;
    {
      const long long* ss = M.seg_cached ? M.seg_s : (const long long*)(A.t.tb.seg_start + M.sb);
      const long long* sc = M.seg_cached ? M.seg_c : (const long long*)(A.t.tb.seg_cnt + M.sb);
      assign_segments<!kTotals>(ss, sc, p1, K, base, vm, v, vnext, sj, hm, pem, rem);
    }

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
    if (lane == 31) S.wtot[wid] = inc;
    __syncthreads();
    if (tid == 0) {
      // carry into the tile (exact fixed point from k_tile_scan), then the fixed-order fold of
      // the warp totals
      const FXV cx = fxv_load(M.carry);
      SVf acc = SVf{from_fx(cx.g, Fg), from_fx(cx.h, Fh), cx.c, 0};
      for (int w = 0; w < kWarps; ++w) { S.wcar[w] = acc; acc = comb(acc, S.wtot[w]); }
    }
    __syncthreads();
    {
      const SVf car = comb(S.wcar[wid], exc);
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        const bool head_before = (hm & ((2u << k) - 1u)) != 0u;
        if (!head_before) { g[k] = car.g + g[k]; h[k] = car.h + h[k]; c[k] = car.c + c[k]; }
      }
    }

    if (kTotals) {
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (((vm & rem) >> k) & 1) {
          const long long s = M.sb + sj[k];
          A.segPG_out[s] = g[k];
          A.segPH_out[s] = h[k];
        }
      }
      __syncthreads();
      continue;
    }

    // ---------------------------------------------------------------- Eq. 2 at run ends
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
        const long long s = M.sb + j;
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
    AM mrun = am_none();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1)) continue;
      AM x;
      x.gain = gn[k]; x.value = v[k];
      x.meta = (ibase + k) | (int)(((dm >> k) & 1) << 12) | (int)(((okm >> k) & 1) << 13);
      x.f = ((hm >> k) & 1) || (tid == 0 && k == 0);
      mrun = am_comb(mrun, x);
    }
    AM minc = mrun;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const AM y = shfl_up(minc, o);
      if (lane >= o) minc = am_comb(y, minc);
    }
    AM mexc = shfl_up(minc, 1);
    if (lane == 0) mexc = am_none();
    if (lane == 31) S.mtot[wid] = minc;
    __syncthreads();
    if (tid == 0) {
      AM acc = am_none();
      for (int w = 0; w < kWarps; ++w) { S.mcar[w] = acc; acc = am_comb(acc, S.mtot[w]); }
    }
    __syncthreads();
    {
      AM r = am_comb(S.mcar[wid], mexc);
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (!((vm >> k) & 1)) continue;
        AM x;
        x.gain = gn[k]; x.value = v[k];
        x.meta = (ibase + k) | (int)(((dm >> k) & 1) << 12) | (int)(((okm >> k) & 1) << 13);
        x.f = ((hm >> k) & 1) || (tid == 0 && k == 0);
        r = am_comb(r, x);
        if (((pem >> k) & 1) && am_valid(r)) S.win[r.meta & 0xfff] = 1;
      }
    }
    __syncthreads();
#pragma unroll
    for (int k = 0; k < kItems; ++k) {
      if (!((vm >> k) & 1) || !S.win[ibase + k]) continue;
      S.win[ibase + k] = 0;
      const int j = sj[k];
      const long long s = M.sb + j;
      Rec r;
      r.gain = gn[k];
      r.value = v[k];
      r.attr = A.t.a_base + M.a;
      r.dir = (dm >> k) & 1;
      r.node = j;
      r.epoch = epoch;
      r.shard = A.shard;
      r.pos = base + k;
      if (r.dir) {
        const int cM = A.nodes.cnt[j] - (int)A.t.tb.seg_cnt[s];
        r.GL = g[k] + (A.nodes.G[j] - A.segPG[s]);
        r.HL = h[k] + (A.nodes.H[j] - A.segPH[s]);
        r.cntL = c[k] + cM;
      } else {
        r.GL = g[k]; r.HL = h[k]; r.cntL = c[k];
      }
      int slot = kPieceList;
      if (cta_table) slot = atomicAdd(&S.npw, 1);
      if (slot < kPieceList) {
        S.pw[slot] = r;
      } else {
        const int gs = atomicAdd(A.nrec, 1);
        A.rec[gs] = r;
        atomicMax(A.gkey + j, gain_key(r.gain));
      }
    }
    __syncthreads();
  }
  // flush the CTA's node bests
  if (cta_table) {
    __syncthreads();
    if (tid == 0 && S.npw) cta_merge(S);
    __syncthreads();
    for (int j = tid; j < K; j += kThreads) {
      if (S.cg[j]) {
        const int gs = atomicAdd(A.nrec, 1);
        A.rec[gs] = S.cb[j];
        atomicMax(A.gkey + j, S.cg[j]);
      }
    }
  }
}

// ============================================================================ a8: partition
// Per tile: (high, low) counts; with missing values also the per-segment counts.
__global__ void __launch_bounds__(kThreads, kLiteBlocks) k_part_count(PartArgs A, int counted) {
  __shared__ TabCache tc;
  __shared__ TileMeta sm;
  __shared__ unsigned ws[kWarps];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int K = *A.t.Kp;
  const int T = *A.t.tb.T;
  if (K == 0 || T == 0) return;
  tab_load(tc, A.t);
  __syncthreads();
  for (int t = blockIdx.x; t < T; t += gridDim.x) {
    if (tid == 0) tile_meta(tc, A.t, K, t, sm);
    __syncthreads();
    const long long p1 = sm.p1;
    const long long base = sm.p0 + (long long)tid * kItems;
    unsigned vm = 0, loc = 0;
    uint8_t sd[kItems];
    if (base < p1) {
      const int4 i0 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base));
      const int4 i1 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base + 4));
      const int id[kItems] = {i0.x, i0.y, i0.z, i0.w, i1.x, i1.y, i1.z, i1.w};
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        sd[k] = 0;
        if (base + k < p1) { vm |= 1u << k; sd[k] = __ldg(A.side + id[k]); }
        loc += sd[k] == 1 ? 1u : (sd[k] == 2 ? (1u << 16) : 0u);
      }
    } else {
#pragma unroll
      for (int k = 0; k < kItems; ++k) sd[k] = 0;
    }
    if (counted && vm) {
      int sj[kItems];
      unsigned hm, pem, rem;
      float vd[kItems];
      assign_segments<false>((const long long*)(A.t.tb.seg_start + sm.sb), (const long long*)(A.t.tb.seg_cnt + sm.sb),
                             p1, K, base, vm, vd, 0.f, sj, hm, pem, rem);
      int cur = -1, ch = 0, cl = 0;
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        if (!((vm >> k) & 1)) continue;
        if (sj[k] != cur) {
          if (cur >= 0) {
            if (ch) atomicAdd(A.segH + sm.sb + cur, ch);
            if (cl) atomicAdd(A.segL + sm.sb + cur, cl);
          }
          cur = sj[k]; ch = cl = 0;
        }
        ch += sd[k] == 1;
        cl += sd[k] == 2;
      }
      if (cur >= 0) {
        if (ch) atomicAdd(A.segH + sm.sb + cur, ch);
        if (cl) atomicAdd(A.segL + sm.sb + cur, cl);
      }
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) loc += __shfl_xor_sync(0xffffffffu, loc, o);
    if (lane == 0) ws[wid] = loc;
    __syncthreads();
    if (tid == 0) {
      unsigned x = 0;
      for (int w = 0; w < kWarps; ++w) x += ws[w];
      A.tcnt[t] = x;
    }
    __syncthreads();
  }
}

// One warp per attribute: exclusive scan of the tile counts within the attribute list.
__global__ void __launch_bounds__(256) k_part_tscan(PartArgs A) {
  const int K = *A.t.Kp;
  if (K == 0) return;
  const int lane = threadIdx.x & 31;
  const int warps = gridDim.x * (blockDim.x >> 5);
  for (int a = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5); a < A.t.m; a += warps) {
    const int t0 = A.t.tb.tile_start[a], t1 = A.t.tb.tile_start[a + 1];
    unsigned long long carry = 0;
    for (int base = t0; base < t1; base += 32) {
      const int t = base + lane;
      unsigned long long x = 0;
      if (t < t1) { const unsigned c = A.tcnt[t]; x = (unsigned long long)(c & 0xffffu) | ((unsigned long long)(c >> 16) << 32); }
      unsigned long long inc = x;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
      }
      if (t < t1) A.tpre[t] = carry + inc - x;
      carry += __shfl_sync(0xffffffffu, inc, 31);
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

// Single thread block: places every child segment (stable, attribute-major, children in heap
// order) and builds the next level's attribute/tile/segment tables.
__global__ void __launch_bounds__(1024) k_part_plan(PlanArgs A) {
  const int K = *A.Kp, Kn = *A.Knp, m = A.m;
  if (!A.counted) {
    // no missing values: every instance of a node is present in every attribute list
    for (long long s = threadIdx.x; s < (long long)m * K; s += blockDim.x) {
      const int c = A.cidx[s % K];
      A.segH[s] = c >= 0 ? A.ncnt[c] : 0;
      A.segL[s] = c >= 0 ? A.ncnt[c + 1] : 0;
    }
    __syncthreads();
  }
  // per attribute: exclusive (high, low) counts before each segment, and the child list length
  for (int a = threadIdx.x; a < m; a += blockDim.x) {
    unsigned long long pre = 0;
    long long L = 0;
    for (int j = 0; j < K; ++j) {
      const long long s = (long long)a * K + j;
      const unsigned hi = (unsigned)A.segH[s], lo = (unsigned)A.segL[s];
      A.seg_pre[s] = pre;
      pre += (unsigned long long)hi | ((unsigned long long)lo << 32);
      if (A.cidx[j] >= 0) L += (long long)hi + lo;
    }
    A.len_tmp[a] = L;
    A.nxt.col_len[a] = L;
  }
  __syncthreads();
  unsigned long long cpos = 0, ctile = 0, t1, t2;
  for (int base = 0; base < m; base += blockDim.x) {
    const int a = base + threadIdx.x;
    const unsigned long long L = a < m ? (unsigned long long)A.len_tmp[a] : 0ull;
    const unsigned long long ep = block_exscan_u64((L + 3) & ~3ull, t1);
    const unsigned long long et = block_exscan_u64((L + kTile - 1) / kTile, t2);
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

// Stable scatter ("Scatter"): out(e) = out_base(seg, side) + rank of e among the
// segment's same-side entries = C_side(e) - C_side(seg start), C counted within the attribute.
__global__ void __launch_bounds__(kThreads, kLiteBlocks) k_part_scatter(PartArgs A) {
  __shared__ TabCache tc;
  __shared__ TileMeta sm;
  __shared__ unsigned ws[kWarps];
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const int K = *A.t.Kp;
  const int T = *A.t.tb.T;
  if (K == 0 || T == 0) return;
  tab_load(tc, A.t);
  __syncthreads();
  for (int t = blockIdx.x; t < T; t += gridDim.x) {
    if (tid == 0) tile_meta(tc, A.t, K, t, sm);
    __syncthreads();
    const long long p1 = sm.p1;
    const long long base = sm.p0 + (long long)tid * kItems;
    unsigned vm = 0, loc = 0;
    float v[kItems];
    int id[kItems];
    uint8_t sd[kItems];
    if (base < p1) {
      const int4 i0 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base));
      const int4 i1 = __ldcs(reinterpret_cast<const int4*>(A.t.ins + base + 4));
      const float4 v0 = __ldcs(reinterpret_cast<const float4*>(A.t.val + base));
      const float4 v1 = __ldcs(reinterpret_cast<const float4*>(A.t.val + base + 4));
      id[0] = i0.x; id[1] = i0.y; id[2] = i0.z; id[3] = i0.w; id[4] = i1.x; id[5] = i1.y; id[6] = i1.z; id[7] = i1.w;
      v[0] = v0.x; v[1] = v0.y; v[2] = v0.z; v[3] = v0.w; v[4] = v1.x; v[5] = v1.y; v[6] = v1.z; v[7] = v1.w;
#pragma unroll
      for (int k = 0; k < kItems; ++k) {
        sd[k] = 0;
        if (base + k < p1) { vm |= 1u << k; sd[k] = __ldg(A.side + id[k]); }
        loc += sd[k] == 1 ? 1u : (sd[k] == 2 ? (1u << 16) : 0u);
      }
    } else {
#pragma unroll
      for (int k = 0; k < kItems; ++k) { sd[k] = 0; v[k] = 0.f; id[k] = 0; }
    }
    int sj[kItems];
    unsigned hm, pem, rem;
    assign_segments<false>((const long long*)(A.t.tb.seg_start + sm.sb), (const long long*)(A.t.tb.seg_cnt + sm.sb),
                           p1, K, base, vm, v, 0.f, sj, hm, pem, rem);
    unsigned inc = loc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned y = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += y;
    }
    if (lane == 31) ws[wid] = inc;
    __syncthreads();
    unsigned wex = 0;
    for (int w = 0; w < wid; ++w) wex += ws[w];
    unsigned ex = wex + inc - loc;
    const unsigned long long tp = A.tpre[t];
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

template <class KernelT>
unsigned grid_for(KernelT kern, size_t smem, int sms) {
  if (smem) GBDT_CUDA(cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  GBDT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kThreads, smem));
  if (occ < 1) fail(GBDT_E_CUDA, "kernel does not fit on an SM");
  return (unsigned)(occ * sms);
}

size_t sf_smem(int hmode) {
  size_t b = (sizeof(SFSmem) + 127) & ~size_t(127);
  if (hmode == kHGather) b += sizeof(double) * kStages * kTile;
  return b;
}

template <int HM>
void launch_sf(const SplitArgs& A, bool missing, unsigned grid, cudaStream_t st) {
  if (missing) k_sf<HM, true, false><<<grid, kThreads, sf_smem(HM), st>>>(A);
  else k_sf<HM, false, false><<<grid, kThreads, sf_smem(HM), st>>>(A);
}

}  // namespace

void LevelKernels::init(int device) {
  GBDT_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, device));
  grid_sf[0][0] = grid_for(k_sf<0, false, false>, sf_smem(0), sms);
  grid_sf[0][1] = grid_for(k_sf<0, true, false>, sf_smem(0), sms);
  grid_sf[1][0] = grid_for(k_sf<1, false, false>, sf_smem(1), sms);
  grid_sf[1][1] = grid_for(k_sf<1, true, false>, sf_smem(1), sms);
  grid_sf[2][0] = grid_for(k_sf<2, false, false>, sf_smem(2), sms);
  grid_sf[2][1] = grid_for(k_sf<2, true, false>, sf_smem(2), sms);
  grid_tot[0] = grid_for(k_sf<0, true, true>, sf_smem(0), sms);
  grid_tot[1] = grid_for(k_sf<1, true, true>, sf_smem(1), sms);
  grid_tot[2] = grid_for(k_sf<2, true, true>, sf_smem(2), sms);
  grid_agg[0] = grid_for(k_tile_agg<0>, 0, sms);
  grid_agg[1] = grid_for(k_tile_agg<1>, 0, sms);
  grid_agg[2] = grid_for(k_tile_agg<2>, 0, sms);
  grid_scatter = grid_for(k_part_scatter, 0, sms);
  grid_count = grid_for(k_part_count, 0, sms);
}

void LevelKernels::tile_prefix(const SplitArgs& A, int hmode, cudaStream_t st) {
  if (hmode == 0) k_tile_agg<0><<<grid_agg[0], kThreads, 0, st>>>(A);
  else if (hmode == 1) k_tile_agg<1><<<grid_agg[1], kThreads, 0, st>>>(A);
  else k_tile_agg<2><<<grid_agg[2], kThreads, 0, st>>>(A);
  GBDT_LAUNCH_CHECK();
  const unsigned g = (unsigned)std::max(1, std::min(A.t.m, sms * 64) / 8 + 1);
  k_tile_scan<<<g, 256, 0, st>>>(A);
  GBDT_LAUNCH_CHECK();
  count_launch(2);
}

void LevelKernels::split_find(const SplitArgs& A, int hmode, bool missing, cudaStream_t st) {
  if (hmode == 0) launch_sf<0>(A, missing, grid_sf[0][missing], st);
  else if (hmode == 1) launch_sf<1>(A, missing, grid_sf[1][missing], st);
  else launch_sf<2>(A, missing, grid_sf[2][missing], st);
  GBDT_LAUNCH_CHECK();
  count_launch();
}

void LevelKernels::seg_totals(const SplitArgs& A, int hmode, cudaStream_t st) {
  if (hmode == 0) k_sf<0, true, true><<<grid_tot[0], kThreads, sf_smem(0), st>>>(A);
  else if (hmode == 1) k_sf<1, true, true><<<grid_tot[1], kThreads, sf_smem(1), st>>>(A);
  else k_sf<2, true, true><<<grid_tot[2], kThreads, sf_smem(2), st>>>(A);
  GBDT_LAUNCH_CHECK();
  count_launch();
}

void LevelKernels::partition(const PartArgs& A, const PlanArgs& P, bool counted, cudaStream_t st) {
  k_part_count<<<grid_count, kThreads, 0, st>>>(A, counted ? 1 : 0);
  GBDT_LAUNCH_CHECK();
  const unsigned g = (unsigned)std::max(1, std::min(A.t.m, sms * 64) / 8 + 1);
  k_part_tscan<<<g, 256, 0, st>>>(A);
  GBDT_LAUNCH_CHECK();
  k_part_plan<<<1, 1024, 0, st>>>(P);
  GBDT_LAUNCH_CHECK();
  k_part_scatter<<<grid_scatter, kThreads, 0, st>>>(A);
  GBDT_LAUNCH_CHECK();
  count_launch(4);
}

}  // namespace gbdt
