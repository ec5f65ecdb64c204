// Feasibility micro-benchmark (not part of the product): can the partition count (an L1TEX-bound
// gather of one bit per entry) run concurrently with the partition scatter (a DRAM-bound stream)
// on the same SMs, so that a pipeline over attribute groups hides the count?  C3 shapes: 308 M
// entries, 11 M instances.  Prints ms for each kernel alone and for the two overlapped on two
// streams, at several grid sizes.
#include <cstdio>
#include <cstdint>
#include <cstdlib>
#include <vector>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { printf("%s:%d %s\n", __FILE__, __LINE__, cudaGetErrorString(e)); exit(1); } } while (0)

constexpr int kChunk = 256;

__global__ void __launch_bounds__(256) k_count(long long c0, long long c1, const int32_t* __restrict__ ins,
                                               const uint32_t* __restrict__ bits, uint8_t* __restrict__ side,
                                               int* __restrict__ ccnt) {
  const int lane = threadIdx.x & 31;
  const long long nw = (long long)gridDim.x * (blockDim.x >> 5);
  for (long long c = c0 + ((long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)); c < c1; c += nw) {
    const long long p0 = c * kChunk;
    int id[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) id[k] = __ldcs(ins + p0 + 32 * k + lane);
    unsigned b[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) b[k] = (__ldg(bits + (id[k] >> 5)) >> (id[k] & 31)) & 1u;
    int cnt = 0;
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      cnt += __popc(__ballot_sync(0xffffffffu, b[k]));
      side[p0 + 32 * k + lane] = (uint8_t)(1 + b[k]);
    }
    if (lane == 0) ccnt[c] = cnt;
  }
}

__global__ void __launch_bounds__(256) k_scatter(long long c0, long long c1, const float* __restrict__ val,
                                                 const int32_t* __restrict__ ins, const double* __restrict__ g,
                                                 const uint8_t* __restrict__ side, const int* __restrict__ cpre,
                                                 float* __restrict__ oval, int32_t* __restrict__ oins,
                                                 double* __restrict__ og, long long nhalf) {
  const int lane = threadIdx.x & 31;
  const long long nw = (long long)gridDim.x * (blockDim.x >> 5);
  for (long long c = c0 + ((long long)blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5)); c < c1; c += nw) {
    const long long p0 = c * kChunk;
    long long hi = cpre[c], lo = nhalf + (p0 - cpre[c]);
#pragma unroll 2
    for (int k = 0; k < 8; ++k) {
      const long long p = p0 + 32 * k + lane;
      const float v = __ldcs(val + p);
      const int32_t i = __ldcs(ins + p);
      const double x = __ldcs(g + p);
      const bool h = __ldcs(side + p) == 2;
      const unsigned bh = __ballot_sync(0xffffffffu, h);
      const unsigned lt = (1u << lane) - 1u;
      const long long d = h ? hi + __popc(bh & lt) : lo + __popc(~bh & lt);
      long long dd = d < 0 ? 0 : d;
      __stcs(oval + dd, v);
      __stcs(oins + dd, i);
      __stcs(og + dd, x);
      hi += __popc(bh);
      lo += 32 - __popc(bh);
    }
  }
}

int main() {
  const long long n = 11000000, N = 308000000ll;
  const long long C = N / kChunk;
  int dev = 0, sms = 0;
  CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  int32_t* ins; float* val; double* g; uint8_t* side; uint32_t* bits; int *ccnt, *cpre;
  float* oval; int32_t* oins; double* og;
  CK(cudaMalloc(&ins, N * 4)); CK(cudaMalloc(&val, N * 4)); CK(cudaMalloc(&g, N * 8));
  CK(cudaMalloc(&side, N)); CK(cudaMalloc(&bits, (n + 31) / 32 * 4));
  CK(cudaMalloc(&ccnt, C * 4)); CK(cudaMalloc(&cpre, C * 4));
  CK(cudaMalloc(&oval, N * 4)); CK(cudaMalloc(&oins, N * 4)); CK(cudaMalloc(&og, N * 8));
  {
    std::vector<int32_t> h(N);
    uint64_t s = 88172645463325252ull;
    for (long long i = 0; i < N; ++i) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; h[i] = (int32_t)(s % n); }
    CK(cudaMemcpy(ins, h.data(), N * 4, cudaMemcpyHostToDevice));
    std::vector<uint32_t> b((n + 31) / 32);
    for (auto& x : b) { s ^= s << 13; s ^= s >> 7; s ^= s << 17; x = (uint32_t)s; }
    CK(cudaMemcpy(bits, b.data(), b.size() * 4, cudaMemcpyHostToDevice));
    std::vector<int> pre(C);
    for (long long c = 0; c < C; ++c) pre[c] = (int)(c * 128);
    CK(cudaMemcpy(cpre, pre.data(), C * 4, cudaMemcpyHostToDevice));
  }
  CK(cudaMemset(val, 0, N * 4)); CK(cudaMemset(g, 0, N * 8));
  k_count<<<sms * 8, 256>>>(0, C, ins, bits, side, ccnt);
  CK(cudaDeviceSynchronize());
  cudaStream_t s1, s2;
  CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
  CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, f1, f2;
  CK(cudaEventCreate(&e0)); CK(cudaEventCreate(&e1)); CK(cudaEventCreate(&f1)); CK(cudaEventCreate(&f2));
  auto timeit = [&](auto fn) {
    float best = 1e9;
    for (int r = 0; r < 5; ++r) {
      CK(cudaDeviceSynchronize());
      CK(cudaEventRecord(e0, s1));
      CK(cudaStreamWaitEvent(s2, e0));
      fn();
      CK(cudaEventRecord(f2, s2));
      CK(cudaStreamWaitEvent(s1, f2));
      CK(cudaEventRecord(e1, s1));
      CK(cudaEventSynchronize(e1));
      float ms; CK(cudaEventElapsedTime(&ms, e0, e1));
      if (ms < best) best = ms;
    }
    return best;
  };
  const long long nh = N / 2;
  for (int cg : {2, 4, 8}) {
    for (int sg : {1, 2, 3, 4}) {
      const float tc = timeit([&] { k_count<<<sms * cg, 256, 0, s1>>>(0, C, ins, bits, side, ccnt); });
      const float ts = timeit([&] { k_scatter<<<sms * sg, 256, 0, s1>>>(0, C, val, ins, g, side, cpre, oval, oins, og, nh); });
      const float tch = timeit([&] { k_count<<<sms * cg, 256, 0, s1>>>(0, C / 2, ins, bits, side, ccnt); });
      const float tsh = timeit([&] { k_scatter<<<sms * sg, 256, 0, s1>>>(0, C / 2, val, ins, g, side, cpre, oval, oins, og, nh); });
      const float tov = timeit([&] {
        k_scatter<<<sms * sg, 256, 0, s1>>>(0, C / 2, val, ins, g, side, cpre, oval, oins, og, nh);
        k_count<<<sms * cg, 256, 0, s2>>>(C / 2, C, ins, bits, side, ccnt);
      });
      printf("count grid %d/SM scatter grid %d/SM: count %.3f scatter %.3f | halves: count %.3f scatter %.3f "
             "overlapped %.3f (serial %.3f) -> pipelined level %.3f vs serial %.3f\n",
             cg, sg, tc, ts, tch, tsh, tov, tch + tsh, tch + tov + tsh, tc + ts);
    }
  }
  return 0;
}
