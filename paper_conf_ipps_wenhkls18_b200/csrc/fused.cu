// fused.cu -- dense levels below the root in ONE streaming pass per level.
//
// For data without missing values every (node, attribute) segment of node j holds exactly the
// node's cnt[j] instances, so the partition of level l and the split finding of
// level l+1 can share one read of the level's lists:
//
//   k_fused   persistent CTAs claim 2048-entry tiles in order (a ticket counter) and stream each
//             tile's values, instance ids and g-list into shared memory with TMA 1-D bulk copies
//             (2-stage ring).  Per tile:
//               1. every entry's child side: the node's decision (leaf -> dropped) and, for a
//                  split node, one bit gathered from the instance -> high-child bitmap
//               2. a stable in-tile partition by (segment, side), ranked by a block scan of the
//                  packed side counts: the tile becomes contiguous runs of CHILD entries in child
//                  order (order preserving)
//               3. a segmented prefix sum of (g, h) over those runs (Fig. 1); the
//                  child segment's prefix from earlier tiles arrives through a decoupled look-back
//                  over per-tile records (counts and exact 128-bit fixed-point sums, so any
//                  look-back path gives bit-identical carries)
//               4. Eq. 2 (+lambda per reading R1) at every boundary between two distinct
//                  values of a child segment (run ends), exact IEEE divisions; per
//                  child node argmax in the R12 total order, merged per CTA, flushed once
//               5. the child runs written to the next level's lists (coalesced), unless the
//                  children are the last level that splits
//   k_mark_fused   the instance -> child bits of a level found by k_fused: the winner's child
//             segment is the winner's side of its parent segment in the PARENT level's lists,
//             and the high part of it is every such entry at a parent position <= Rec.pos
//
// Determinism: tiles are attribute-aligned (tile k of an attribute covers its list positions
// [2048 k, 2048 k + 2048) at that level), inside a tile every sum has a fixed association, and
// carries are exact integer sums, so every gain -- hence every tree -- is bit-identical for any
// attribute sharding and any schedule.
#include <algorithm>
#include <climits>

#include "kernels.cuh"

namespace gbdt {
namespace {

constexpr int kFT = 256;            // threads per CTA
constexpr int kFI = 8;              // items per thread (blocked arrangement)
constexpr int kFTile = kFT * kFI;   // entries per tile
constexpr int kFW = kFT / 32;
// One tile in flight per CTA.  A CTA that also held the ticket of its next tile (a 2-stage TMA
// ring) would publish that tile's look-back record a whole tile later than it could, and the tiles
// of its chain behind it would wait (measured: C3 148 vs 49 ms/tree, 84 % of stall samples at the
// barrier behind the look-back).  The load latency is hidden by the other CTAs of the SM instead.
#ifndef GBDT_FUSED_CTAS
#define GBDT_FUSED_CTAS 3
#endif

// The look-back record of one tile: per child side (0 high, 1 low) the entries of its LAST
// segment piece, their exact fixed-point sums, and the value / parent position of the last one.
struct __align__(16) LBSide {
  unsigned long long g_lo, g_hi, h_lo, h_hi;
  long long pos;
  int cnt;
  float val;
};
struct __align__(16) LBRec {
  LBSide s[2];
};
static_assert(sizeof(LBRec) == 96, "look-back record");
constexpr unsigned kLBAgg = 1, kLBInc = 2;
__device__ __forceinline__ LBRec* lb_agg(const FusedArgs& A) { return static_cast<LBRec*>(A.lb_agg_); }
__device__ __forceinline__ LBRec* lb_inc(const FusedArgs& A) { return static_cast<LBRec*>(A.lb_inc_); }

struct FusedSmem {
  float val[kFTile];                // the tile as loaded (TMA), never reordered in place
  int32_t ins[kFTile];
  double g[kFTile];
  unsigned short src[kFTile];       // child order: slot r holds tile entry src[r]
  unsigned long long bar;
  int tile;
  // plan copy
  int off[kFusedMaxK + 1];
  int cidx[kFusedMaxK];
  int offn[2 * kFusedMaxK + 1];
  double cG[2 * kFusedMaxK], cH[2 * kFusedMaxK], cHl[2 * kFusedMaxK], cP[2 * kFusedMaxK];
  // CTA node-best table (children)
  unsigned long long ngk[2 * kFusedMaxK];
  Rec nrec[2 * kFusedMaxK];
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
  double lg[2], lh[2];              // sums of the last piece's two groups
  float lv[2];
  int ls[2];                        // tile entry of the groups' last members
  LBSide ex[2];                     // carry of the first piece (look-back)
};

__device__ __forceinline__ unsigned ld_acquire_u32(const unsigned* p) {
  unsigned v;
  asm volatile("ld.global.acquire.gpu.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release_u32(unsigned* p, unsigned v) {
  asm volatile("st.global.release.gpu.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}

__device__ __forceinline__ unsigned __int128 u128(unsigned long long lo, unsigned long long hi) {
  return ((unsigned __int128)hi << 64) | lo;
}
__device__ __forceinline__ unsigned __int128 warp_sum128(unsigned __int128 v) {
#pragma unroll
  for (int o = 16; o; o >>= 1) {
    const unsigned long long lo = __shfl_xor_sync(0xffffffffu, (unsigned long long)v, o);
    const unsigned long long hi = __shfl_xor_sync(0xffffffffu, (unsigned long long)(v >> 64), o);
    v += u128(lo, hi);
  }
  return v;
}

__device__ __forceinline__ void lb_store(LBRec* dst, const LBSide* s) {
  for (int q = 0; q < 2; ++q) {
    dst->s[q].g_lo = s[q].g_lo; dst->s[q].g_hi = s[q].g_hi;
    dst->s[q].h_lo = s[q].h_lo; dst->s[q].h_hi = s[q].h_hi;
    dst->s[q].pos = s[q].pos; dst->s[q].cnt = s[q].cnt; dst->s[q].val = s[q].val;
  }
}

// Exclusive carry of tile t's first segment piece from the tiles before it (one warp).  Lane i
// inspects tile t-1-i; the chain ends at the closest tile whose record is inclusive (the tile in
// which the segment starts publishes an inclusive record at once).
// Only tiles >= tmin (the tile holding the segment's start, whose record is inclusive) are read:
// with tickets dealt round-robin over the attributes, tiles before tmin may belong to a later
// ticket, and waiting on them could deadlock.
__device__ void lookback(const FusedArgs& A, int t, int tmin, unsigned ep, LBSide* out, int lane) {
  unsigned __int128 G[2] = {0, 0}, H[2] = {0, 0};
  long long cnt[2] = {0, 0};
  float lv[2] = {0.f, 0.f};
  long long lp[2] = {0, 0};
  bool have[2] = {false, false};
  int base = t - 1;
  while (true) {
    const int idx = base - lane;
    unsigned s = (ep << 2) | kLBInc;
    if (idx >= tmin) {
      do {
        s = ld_acquire_u32(A.lb_status + idx);
      } while ((s >> 2) != ep || (s & 3u) == 0u);
    }
    const bool inc = (s & 3u) == kLBInc;
    const unsigned incm = __ballot_sync(0xffffffffu, inc);
    const int lim = incm ? __ffs(incm) - 1 : 31;
    const bool use = lane <= lim && idx >= tmin;
    const LBRec* src = use ? ((inc ? lb_inc(A) : lb_agg(A)) + idx) : nullptr;
#pragma unroll
    for (int q = 0; q < 2; ++q) {
      unsigned __int128 g = 0, h = 0;
      int c = 0;
      float v = 0.f;
      long long p = 0;
      if (use) {
        const unsigned long long* w = reinterpret_cast<const unsigned long long*>(&src->s[q]);
        g = u128(__ldcg(w + 0), __ldcg(w + 1));
        h = u128(__ldcg(w + 2), __ldcg(w + 3));
        p = (long long)__ldcg(w + 4);
        const unsigned long long cv = __ldcg(w + 5);
        c = (int)(unsigned)cv;
        v = __uint_as_float((unsigned)(cv >> 32));
      }
      const unsigned nz = __ballot_sync(0xffffffffu, use && c > 0);
      if (!have[q] && nz) {  // the last value of this side: the closest tile that has one
        const int l = __ffs(nz) - 1;
        lv[q] = __shfl_sync(0xffffffffu, v, l);
        lp[q] = __shfl_sync(0xffffffffu, p, l);
        have[q] = true;
      }
      int cs = c;
#pragma unroll
      for (int o = 16; o; o >>= 1) cs += __shfl_xor_sync(0xffffffffu, cs, o);
      cnt[q] += cs;
      G[q] += warp_sum128(g);
      H[q] += warp_sum128(h);
    }
    if (incm) break;
    base -= 32;
  }
  if (lane == 0) {
    for (int q = 0; q < 2; ++q) {
      out[q].g_lo = (unsigned long long)G[q]; out[q].g_hi = (unsigned long long)(G[q] >> 64);
      out[q].h_lo = (unsigned long long)H[q]; out[q].h_hi = (unsigned long long)(H[q] >> 64);
      out[q].cnt = (int)cnt[q];
      out[q].val = lv[q];
      out[q].pos = lp[q];
    }
  }
}

__device__ __forceinline__ bool rec_better_f(unsigned long long gk, const Rec& r, unsigned long long gk0, const Rec& r0) {
  return gk > gk0 || (gk == gk0 && tie_key(r.attr, r.value, r.dir) < tie_key(r0.attr, r0.value, r0.dir));
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
  const unsigned long long pol = policy_evict_first();
  // Tickets are dealt round-robin over the attributes (ticket u -> tile u / m of attribute u % m):
  // every attribute's segments form their own look-back chains, so a chain has ~1/m of the tiles
  // in flight and a look-back rarely reads more than one 32-tile window.  Tile index t = a * tpa + k
  // (the look-back predecessor of t is t - 1).
  const int mm = A.m;
  auto tile_of = [&](int u) { return (u % mm) * tpa + u / mm; };
  auto issue = [&](int t) {  // TMA of tile t's lists
    const int a = t / tpa;
    const int q0 = (t - a * tpa) * kFTile;
    const long long p0 = (long long)a * stride + q0;
    const uint32_t n = (uint32_t)((min(kFTile, n_act - q0) + 3) & ~3);
    mbar_arrive_expect_tx(&S.bar, 16u * n);
    tma_load_1d(S.val, A.val + p0, 4u * n, &S.bar, pol);
    tma_load_1d(S.ins, A.ins + p0, 4u * n, &S.bar, pol);
    tma_load_1d(S.g, A.gl + p0, 8u * n, &S.bar, pol);
  };
  if (tid == 0) {
    mbar_init(&S.bar, 1);
    fence_mbar_init();
    const int u = atomicAdd(A.ticket, 1);
    S.tile = u;
    if (u < T) issue(tile_of(u));
  }
  __syncthreads();
  uint32_t phase = 0;
  const int qi = tid * kFI;
  while (true) {
    const int u = S.tile;
    if (u >= T) break;
    const int t = tile_of(u);
    const int a = t / tpa;
    const int q0 = (t - a * tpa) * kFTile;
    const int len = min(kFTile, n_act - q0);
    const long long tbase = (long long)a * stride + q0;
    if (tid == 0) {  // the tile's pieces (parent segments), while the copy is in flight
      int lo = 0, hi = K - 1;
      while (lo < hi) {
        const int mid = (lo + hi + 1) >> 1;
        if (S.off[mid] <= q0) lo = mid; else hi = mid - 1;
      }
      int s = 0;
      S.pq[0] = 0;
      while (S.off[lo + s + 1] < q0 + len) { ++s; S.pq[s] = S.off[lo + s] - q0; }
      S.pq[s + 1] = len;
      S.j0 = lo;
      S.nseg = s + 1;
      S.cont = S.off[lo] < q0 && S.cidx[lo] >= 0;
    }
    mbar_wait(&S.bar, phase);
    phase ^= 1u;
    __syncthreads();
    const int j0 = S.j0, nseg = S.nseg;
    const bool cont = S.cont != 0;

    // ---- 1. child side of every entry; stable in-tile partition by (piece, side) -> src[]
    int sidx[kFI];
    {
      const int4 i0 = reinterpret_cast<const int4*>(S.ins + qi)[0];
      const int4 i1 = reinterpret_cast<const int4*>(S.ins + qi)[1];
      const int id[kFI] = {i0.x, i0.y, i0.z, i0.w, i1.x, i1.y, i1.z, i1.w};
      int s = 0;
      while (s + 1 < nseg && qi >= S.pq[s + 1]) ++s;
      int nb = S.pq[s + 1];
      bool live = S.cidx[j0 + s] >= 0;
      unsigned w[kFI];
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        if (qi + k >= nb && s + 1 < nseg) {
          ++s;
          nb = S.pq[s + 1];
          live = S.cidx[j0 + s] >= 0;
        }
        sidx[k] = (qi + k < len && live) ? s : -1;
        w[k] = sidx[k] >= 0 ? __ldg(A.hbit + (id[k] >> 5)) : 0u;
      }
#pragma unroll
      for (int k = 0; k < kFI; ++k)  // piece index << 2 | side (1 high, 2 low); -1 dropped
        sidx[k] = sidx[k] < 0 ? -1 : ((sidx[k] << 2) | (((w[k] >> (id[k] & 31)) & 1u) ? 1 : 2));
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
          xg[k] = S.g[sr[k]];
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
    // exclusive in-tile prefix per slot (replaces g, h); the last piece's group totals
    {
      double rg = eg, rh = eh;
      int gg = grp0;
#pragma unroll
      for (int k = 0; k < kFI; ++k) {
        const int r = qi + k;
        if (r < nk) {
          if ((gstep >> k) & 1u) { while (r >= S.gb[gg + 1]) ++gg; }
          if ((headm >> k) & 1u) { rg = 0.0; rh = 0.0; }
          const double ng_ = rg + xg[k], nh_ = rh + xh[k];
          if ((gg >> 1) == nseg - 1 && r + 1 == S.gb[gg + 1]) {
            S.lg[gg & 1] = ng_;
            S.lh[gg & 1] = nh_;
            S.lv[gg & 1] = S.val[sr[k]];
            S.ls[gg & 1] = sr[k];
          }
          xg[k] = rg;
          xh[k] = rh;
          rg = ng_;
          rh = nh_;
        }
      }
    }
    __syncthreads();

    // ---- 3. publish this tile's record; look back for the first piece's carry
    if (wid == 0) {
      const int jl = j0 + nseg - 1;
      LBSide rec[2];
      if (lane == 0) {
        const bool live = S.cidx[jl] >= 0;
        for (int q = 0; q < 2; ++q) {
          const int cnt = live ? S.gb[2 * (nseg - 1) + q + 1] - S.gb[2 * (nseg - 1) + q] : 0;
          const __int128 G = cnt ? to_fx(S.lg[q], Fg) : 0, H = cnt ? to_fx(S.lh[q], Fh) : 0;
          rec[q].g_lo = (unsigned long long)G; rec[q].g_hi = (unsigned long long)((unsigned __int128)G >> 64);
          rec[q].h_lo = (unsigned long long)H; rec[q].h_hi = (unsigned long long)((unsigned __int128)H >> 64);
          rec[q].cnt = cnt;
          rec[q].val = cnt ? S.lv[q] : 0.f;
          rec[q].pos = cnt ? tbase + S.ls[q] : 0;
        }
        const bool last_cont = live && S.off[jl] < q0;  // the last piece began in an earlier tile
        lb_store((last_cont ? lb_agg(A) : lb_inc(A)) + t, rec);
        __threadfence();
        st_release_u32(A.lb_status + t, (ep << 2) | (last_cont ? kLBAgg : kLBInc));
      }
      if (cont) {
        lookback(A, t, a * tpa + S.off[j0] / kFTile, ep, S.ex, lane);
        if (lane == 0 && nseg == 1) {  // the first piece is the last one: inclusive = carry + own
          LBSide inc[2];
          for (int q = 0; q < 2; ++q) {
            const unsigned __int128 G = u128(S.ex[q].g_lo, S.ex[q].g_hi) + u128(rec[q].g_lo, rec[q].g_hi);
            const unsigned __int128 H = u128(S.ex[q].h_lo, S.ex[q].h_hi) + u128(rec[q].h_lo, rec[q].h_hi);
            inc[q].g_lo = (unsigned long long)G; inc[q].g_hi = (unsigned long long)(G >> 64);
            inc[q].h_lo = (unsigned long long)H; inc[q].h_hi = (unsigned long long)(H >> 64);
            inc[q].cnt = S.ex[q].cnt + rec[q].cnt;
            inc[q].val = rec[q].cnt ? rec[q].val : S.ex[q].val;
            inc[q].pos = rec[q].cnt ? rec[q].pos : S.ex[q].pos;
          }
          lb_store(lb_inc(A) + t, inc);
          __threadfence();
          st_release_u32(A.lb_status + t, (ep << 2) | kLBInc);
        }
      } else if (lane < 2) {
        S.ex[lane].g_lo = S.ex[lane].g_hi = S.ex[lane].h_lo = S.ex[lane].h_hi = 0ull;
        S.ex[lane].cnt = 0; S.ex[lane].val = 0.f; S.ex[lane].pos = 0;
      }
    }
    __syncthreads();

    // ---- 4. candidates: the boundary before every child entry whose predecessor in its child
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
      if (qi > gs) { pv = S.val[S.src[qi - 1]]; prev = true; }
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
          const float cv = S.val[sr[k]];
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
      rc.value = ps >= 0 ? S.val[ps] : S.ex[q].val;
      rc.pos = ps >= 0 ? tbase + ps : S.ex[q].pos;
      rc.attr = A.a_base + a;
      rc.dir = 0;
      rc.node = c;
      rc.epoch = (int)ep;
      rc.shard = A.shard;
      if (rec_better_f(rkey[i], rc, S.ngk[c], S.nrec[c])) {  // one writer per child node per tile
        S.nrec[c] = rc;
        S.ngk[c] = rkey[i];
      }
    }
    // ---- 5. child runs -> the next level's lists (coalesced: 32 consecutive slots per warp)
    if (kWrite) {
      int gg = -1, gn = 0;
      long long dbase = 0;
      for (int r = tid; r < nk; r += kFT) {
        if (r >= gn) {
          if (gg < 0) gg = 0;
          while (r >= S.gb[gg + 1]) ++gg;
          gn = S.gb[gg + 1];
          const int s = gg >> 1, q = gg & 1;
          dbase = (long long)a * stride_n + S.offn[S.cidx[j0 + s] + q] + ((s == 0 && cont) ? S.ex[q].cnt : 0) -
                  S.gb[gg];
        }
        const int e = S.src[r];
        __stcs(A.val_out + dbase + r, S.val[e]);
        __stcs(A.ins_out + dbase + r, S.ins[e]);
        __stcs(A.g_out + dbase + r, S.g[e]);
      }
    }
    __syncthreads();  // the tile and its scratch are free
    if (tid == 0) {
      const int u2 = atomicAdd(A.ticket, 1);
      S.tile = u2;
      if (u2 < T) {
        fence_proxy_async();
        issue(tile_of(u2));
      }
    }
    __syncthreads();
  }
  // flush the CTA's node bests (R12 merge across CTAs by k_pick_tie / k_pick_best)
  for (int c = tid; c < Kn; c += kFT) {
    if (S.ngk[c]) {
      const int gs = atomicAdd(A.nrec, 1);
      A.rec[gs] = S.nrec[c];
      atomicMax(A.gkey + c, S.ngk[c]);
    }
  }
}

// One block: the level's segment offsets, child offsets / parents, tile count; resets the ticket.
__global__ void k_fused_plan(FusedPlan* P, NodeTab cur, NodeTab nxt, const int32_t* __restrict__ cidx,
                             const int* __restrict__ epoch, int m, int* ticket, unsigned long long* lent, int lvl) {
  if (threadIdx.x != 0) return;
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
  *ticket = 0;
  if (lent) lent[lvl + 1] += (unsigned long long)on * (unsigned long long)m;
}

// Instance -> non-default-side bits of the splits found by k_fused (level l+1), marked from the
// parent level l's lists: child c's entries are the entries of its parent's segment on c's side
// (high child: even c), in order; the high part of c's split is those at positions <= pos.
__global__ void k_mark_fused(const FusedPlan* __restrict__ P, const int32_t* __restrict__ Kp,
                             const int32_t* __restrict__ cidx_now, const Rec* __restrict__ winner, int shard,
                             int a_base, const int32_t* __restrict__ ins, const uint32_t* __restrict__ hbit,
                             uint8_t* __restrict__ bits) {
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
    if (high != w.dir) bits[i] = 1;
  }
}

unsigned g_fused_grid[2][2] = {{0, 0}, {0, 0}};

template <int HM, bool W>
void set_fused(int sms) {
  const size_t smem = sizeof(FusedSmem);
  GBDT_CUDA(cudaFuncSetAttribute(k_fused<HM, W>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int occ = 0;
  GBDT_CUDA(cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k_fused<HM, W>, kFT, smem));
  if (occ < 1) fail(GBDT_E_CUDA, "k_fused does not fit on an SM");
  g_fused_grid[HM][W ? 1 : 0] = (unsigned)(occ * sms);
}

}  // namespace

size_t fused_lb_bytes(int64_t max_tiles) { return (size_t)max_tiles * (sizeof(LBRec) * 2 + 4); }
int64_t fused_tiles(int64_t n, int m) { return (int64_t)m * ((n + kFTile - 1) / kFTile); }

void fused_init(int sms) {
  set_fused<kHConst2, true>(sms);
  set_fused<kHConst2, false>(sms);
  set_fused<kHFromG, true>(sms);
  set_fused<kHFromG, false>(sms);
}

unsigned fused_grid(int hmode) { return std::max(g_fused_grid[hmode][0], g_fused_grid[hmode][1]); }

void fused_plan(FusedPlan* P, const NodeTab& cur, const NodeTab& nxt, const int32_t* cidx, const int* epoch, int m,
                int* ticket, unsigned long long* lent, int lvl, cudaStream_t st) {
  k_fused_plan<<<1, 32, 0, st>>>(P, cur, nxt, cidx, epoch, m, ticket, lent, lvl);
  GBDT_LAUNCH_CHECK();
  count_launch();
}

void fused_pass(const FusedArgs& A, int hmode, bool write, cudaStream_t st) {
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
  count_launch();
}

void fused_mark(const FusedPlan* P, const int32_t* Kp, const int32_t* cidx, const Rec* winner, int shard, int a_base,
                const int32_t* ins, const uint32_t* hbit, uint8_t* bits, int64_t n, int Kl, int sms, cudaStream_t st) {
  dim3 grid((unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256 * (int64_t)Kl), (int64_t)sms * 4)),
            (unsigned)Kl);
  k_mark_fused<<<grid, 256, 0, st>>>(P, Kp, cidx, winner, shard, a_base, ins, hbit, bits);
  GBDT_LAUNCH_CHECK();
  count_launch();
}

}  // namespace gbdt
