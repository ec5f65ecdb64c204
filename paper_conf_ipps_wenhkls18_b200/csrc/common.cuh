// common.cuh -- device helpers shared by the sm_100a kernels of libgbdt.so.
// (Product code; nothing here is shared with oracle/.)
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "internal.h"

namespace gbdt {

// ----------------------------------------------------------------------------- launch config
constexpr int kThreads = 256;          // threads per tile CTA (8 warps)
constexpr int kItems = 8;              // entries per thread, blocked arrangement
constexpr int kTile = kThreads * kItems;  // 2048 entries per tile (attribute-aligned)
constexpr int kWarps = kThreads / 32;
constexpr int kChunk = 32 * kItems;    // 256 entries: the unit of one warp (8 per tile)

// ----------------------------------------------------------------------------- memory order
__device__ __forceinline__ int ld_acquire(const int* p) {
  int v;
  asm volatile("ld.global.acquire.gpu.b32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}
__device__ __forceinline__ void st_release(int* p, int v) {
  asm volatile("st.global.release.gpu.b32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ double ldcg(const double* p) { return __ldcg(p); }
__device__ __forceinline__ unsigned long long ld_acquire_u64(const unsigned long long* p) {
  unsigned long long v;
  asm volatile("ld.global.acquire.gpu.b64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
  return v;
}

// ----------------------------------------------------------------------------- TMA / mbarrier
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(unsigned long long* b, uint32_t cnt) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(cnt) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
// orders this thread's earlier generic-proxy smem accesses before later async-proxy (TMA) ones
__device__ __forceinline__ void fence_proxy_async() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(unsigned long long* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ bool mbar_try_wait(unsigned long long* b, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      " selp.b32 %0, 1, 0, p;\n}"
      : "=r"(ok)
      : "r"(smem_u32(b)), "r"(parity)
      : "memory");
  return ok != 0;
}
__device__ __forceinline__ void mbar_wait(unsigned long long* b, uint32_t parity) {
  while (!mbar_try_wait(b, parity)) {
  }
}
__device__ __forceinline__ unsigned long long policy_evict_first() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ unsigned long long policy_evict_last() {
  unsigned long long p;
  asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
// 1-D bulk copy global -> shared (TMA engine, UBLKCP); completion counted on the mbarrier.
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes,
                                            unsigned long long* bar, unsigned long long pol) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1], %2, [%3], %4;" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar)), "l"(pol)
      : "memory");
}
// read-only load that L2 should keep (gathered per-instance gradients)
__device__ __forceinline__ double ld_keep(const double* p, unsigned long long pol) {
  double v;
  asm volatile("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(p), "l"(pol));
  return v;
}
// per-thread async gathers (LDGSTS)
__device__ __forceinline__ void cp_async8(void* dst, const void* src, unsigned long long pol) {
  asm volatile("cp.async.ca.shared.global.L2::cache_hint [%0], [%1], 8, %2;" ::"r"(smem_u32(dst)), "l"(src),
               "l"(pol)
               : "memory");
}
__device__ __forceinline__ void cp_async4(void* dst, const void* src) {
  asm volatile("cp.async.ca.shared.global [%0], [%1], 4;" ::"r"(smem_u32(dst)), "l"(src) : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() {
  asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory");
}

// ----------------------------------------------------------------------------- order keys
// fp64 -> u64 such that unsigned order == numeric order (no NaN reaches here). 0 = "empty".
__device__ __forceinline__ unsigned long long gain_key(double g) {
  if (g == 0.0) g = 0.0;  // -0.0 and +0.0 compare equal (R12 reading: gains, not bit patterns)
  long long b = __double_as_longlong(g);
  return b < 0 ? ~(unsigned long long)b : ((unsigned long long)b | 0x8000000000000000ull);
}
// inverse of gain_key for a non-empty key
__device__ __forceinline__ double key_gain(unsigned long long k) {
  return __longlong_as_double((long long)((k & 0x8000000000000000ull) ? (k & 0x7fffffffffffffffull) : ~k));
}
// fp32 -> u32 ascending order key
__device__ __forceinline__ unsigned int fkey(float v) {
  unsigned int b = __float_as_uint(v);
  return (b & 0x80000000u) ? ~b : (b | 0x80000000u);
}
// tie key, smaller wins: attr asc, value desc, dir low(0) before high(1)   (R12)
__device__ __forceinline__ unsigned long long tie_key(int attr, float value, int dir) {
  return ((unsigned long long)(unsigned)attr << 33) | ((unsigned long long)(~fkey(value)) << 1) |
         (unsigned long long)(dir & 1);
}

// ----------------------------------------------------------------------------- Eq. 2
// gain = 1/2 [GL^2/(HL+l) + GR^2/(HR+l) - G^2/(H+l)] with GR = G-GL, HR = H-HL (R1).
// Every op is an explicitly rounded IEEE fp64 op (no FMA contraction) so that the arithmetic is
// the same sequence of roundings the definition states.
__device__ __forceinline__ double eq2_gain(double GL, double HL, double G, double H, double lam,
                                           double parent_term) {
  double GR = __dsub_rn(G, GL), HR = __dsub_rn(H, HL);
  double t1 = __ddiv_rn(__dmul_rn(GL, GL), __dadd_rn(HL, lam));
  double t2 = __ddiv_rn(__dmul_rn(GR, GR), __dadd_rn(HR, lam));
  double g = __dmul_rn(0.5, __dsub_rn(__dadd_rn(t1, t2), parent_term));
  return g == 0.0 ? 0.0 : g;
}
__device__ __forceinline__ double parent_term(double G, double H, double lam) {
  return __ddiv_rn(__dmul_rn(G, G), __dadd_rn(H, lam));
}

// ----------------------------------------------------------------------------- RLE chunk index
// Run o covers list positions [P, P+L) of attribute a: record it as the run of every chunk whose
// first entry it holds (chunk starts are col_start[a] + 256 k).
__device__ __forceinline__ void fill_run_chunks(int32_t* run_chunk, const Tables& tb, int a, long long P,
                                                long long L, int o) {
  const long long cs = tb.col_start[a];
  const long long k0 = (P - cs + kChunk - 1) / kChunk;
  const long long c0 = tb.chunk_start[a];
  for (long long q = cs + k0 * kChunk; q < P + L; q += kChunk) run_chunk[c0 + (q - cs) / kChunk] = o;
}

// ============================================================================ exact fixed point
// x -> trunc(x * 2^F) as a 128-bit integer.  A pure function of x, and integer addition is
// associative, so sums of converted values are bit-identical in any order.
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
// ----------------------------------------------------------------------------- hessian
// Gradient storage mode of the split-find kernels:
//   0: squared loss, h == 2 (only g is gathered)
//   1: logistic loss with 0/1 labels, h = max(q(1-q), 1e-16), q = g + [g < 0] (K1)
//   2: general: h gathered too
enum { kHConst2 = 0, kHFromG = 1, kHGather = 2 };
template <int HMODE>
__device__ __forceinline__ double hess_of(double g) {
  if (HMODE == kHConst2) return 2.0;
  // logistic, 0/1 labels: g = p - y with p in [0,1], so |g| is 1 - p (y = 1) or p (y = 0) and
  // h = |g| (1 - |g|) = p (1 - p) (K1); |g| is an operand modifier, no select
  const double a = fabs(g);
  const double hh = __dmul_rn(a, __dsub_rn(1.0, a));
  // max(hh, 1e-16); hh is never NaN (q in [0, 1]), so a plain compare-select (no fmax NaN rules)
  double r;
  asm("{\n .reg .pred p;\n setp.lt.f64 p, %1, 0d3C9CD2B297D889BC;\n selp.f64 %0, 0d3C9CD2B297D889BC, %1, p;\n}"
      : "=d"(r) : "d"(hh));
  return r;
}

// ----------------------------------------------------------------------------- scan value
struct SV {
  double g, h;
  int c;
};
__device__ __forceinline__ SV sv_zero() { return SV{0.0, 0.0, 0}; }
// left (+) right, left-to-right association
__device__ __forceinline__ SV sv_add(const SV& a, const SV& b) {
  return SV{__dadd_rn(a.g, b.g), __dadd_rn(a.h, b.h), a.c + b.c};
}

// ----------------------------------------------------------------------------- tree traversal
// Value of attribute a in CSR row i (binary search; rows have strictly increasing indices).
// NaN = missing; -0.0 reads as +0.0 as in the layout.
__device__ __forceinline__ bool csr_lookup(const int64_t* indptr, const int32_t* indices, const float* values,
                                           int64_t i, int a, float& x) {
  int64_t lo = indptr[i], hi = indptr[i + 1];
  while (lo < hi) {
    const int64_t mid = lo + ((hi - lo) >> 1);
    if (indices[mid] < a) lo = mid + 1; else hi = mid;
  }
  if (lo < indptr[i + 1] && indices[lo] == a) {
    const float v = values[lo];
    if (isnan(v)) return false;
    x = v == 0.0f ? 0.0f : v;
    return true;
  }
  return false;
}

// Leaf weight of row i in tree T (heap order): present x >= split_value goes to the high child
// 2k+1, else 2k+2; missing follows default_left (reading R11).
__device__ __forceinline__ double tree_leaf_weight(const gbdt_node* T, const int64_t* indptr, const int32_t* indices,
                                                   const float* values, int64_t i) {
  int64_t k = 0;
  while (!T[k].is_leaf) {
    float x;
    const bool high = csr_lookup(indptr, indices, values, i, T[k].attr, x) ? (x >= T[k].split_value)
                                                                          : (T[k].default_left != 0);
    k = high ? 2 * k + 1 : 2 * k + 2;
  }
  return T[k].weight;
}

}  // namespace gbdt
