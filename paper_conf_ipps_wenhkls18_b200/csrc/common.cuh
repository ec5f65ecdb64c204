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

// ----------------------------------------------------------------------------- order keys
// fp64 -> u64 such that unsigned order == numeric order (no NaN reaches here). 0 = "empty".
__device__ __forceinline__ unsigned long long gain_key(double g) {
  if (g == 0.0) g = 0.0;  // -0.0 and +0.0 compare equal (R12 reading: gains, not bit patterns)
  long long b = __double_as_longlong(g);
  return b < 0 ? ~(unsigned long long)b : ((unsigned long long)b | 0x8000000000000000ull);
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

}  // namespace gbdt
