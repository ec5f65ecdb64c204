// layout.cu -- a1: attribute-major layout build (load time, once per dataset; P:36, P:80-112,
// P:238 "compressed data can be used for multiple times").
//
// CSR rows -> per attribute, present entries sorted by value DESCENDING, ties by
// ascending instance id (reading R9), NaN dropped as missing, -0.0 -> +0.0.  Done with
// one stable LSD radix sort of the composite key (local attr << 32 | ~orderkey(value)) whose
// payload is the instance id: stability keeps the CSR (ascending id) order inside equal keys.
// Each attribute list starts at a 16-byte aligned position (padded to 4 entries) so tiles can
// use 128-bit loads.
#include <algorithm>
#include <cstring>

#include "common.cuh"

namespace gbdt {

namespace {

constexpr int kRadixThreads = 256;
constexpr int kRadixBits = 8;
constexpr int kRadixBins = 1 << kRadixBits;

// Warp per CSR row: emits the sort key and the instance id of every stored entry.
__global__ void k_make_keys(int64_t n, const int64_t* __restrict__ indptr,
                            const int32_t* __restrict__ indices, const float* __restrict__ values,
                            int32_t a_begin, int32_t a_end, unsigned long long* __restrict__ keys,
                            uint32_t* __restrict__ ids) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x / 32);
  const unsigned long long sentinel = (unsigned long long)(uint32_t)(a_end - a_begin) << 32;
  for (int64_t i = (int64_t)blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5); i < n; i += warps) {
    const int64_t lo = indptr[i], hi = indptr[i + 1];
    for (int64_t p = lo + lane; p < hi; p += 32) {
      const int a = indices[p];
      float v = values[p];
      unsigned long long k = sentinel;
      if (a >= a_begin && a < a_end && !isnan(v)) {
        if (v == 0.0f) v = 0.0f;  // -0.0 -> +0.0 so that radix order agrees with float equality
        k = ((unsigned long long)(uint32_t)(a - a_begin) << 32) | (unsigned long long)(~fkey(v));
      }
      keys[p] = k;
      ids[p] = (uint32_t)i;
    }
  }
}

__global__ void k_radix_hist(int64_t N, int64_t chunk, int shift,
                             const unsigned long long* __restrict__ keys,
                             uint32_t* __restrict__ hist /* [bins][blocks] */) {
  __shared__ uint32_t h[kRadixBins];
  for (int i = threadIdx.x; i < kRadixBins; i += blockDim.x) h[i] = 0;
  __syncthreads();
  const int64_t b0 = (int64_t)blockIdx.x * chunk, b1 = min(N, b0 + chunk);
  for (int64_t p = b0 + threadIdx.x; p < b1; p += blockDim.x)
    atomicAdd(&h[(keys[p] >> shift) & (kRadixBins - 1)], 1u);
  __syncthreads();
  for (int i = threadIdx.x; i < kRadixBins; i += blockDim.x) hist[(int64_t)i * gridDim.x + blockIdx.x] = h[i];
}

// Single-CTA exclusive scan of n uint32 counts (n = bins * blocks, a few hundred thousand).
__global__ void k_scan_u32(int64_t n, uint32_t* __restrict__ a) {
  __shared__ uint32_t warp_sums[32];
  __shared__ uint32_t carry;
  if (threadIdx.x == 0) carry = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  for (int64_t base = 0; base < n; base += blockDim.x) {
    const int64_t i = base + threadIdx.x;
    uint32_t x = i < n ? a[i] : 0u, incl = x;
    for (int o = 1; o < 32; o <<= 1) {
      uint32_t y = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += y;
    }
    if (lane == 31) warp_sums[w] = incl;
    __syncthreads();
    if (w == 0) {
      uint32_t s = lane < nw ? warp_sums[lane] : 0u, si = s;
      for (int o = 1; o < 32; o <<= 1) {
        uint32_t y = __shfl_up_sync(0xffffffffu, si, o);
        if (lane >= o) si += y;
      }
      if (lane < nw) warp_sums[lane] = si - s;
    }
    __syncthreads();
    const uint32_t c = carry;
    if (i < n) a[i] = c + warp_sums[w] + incl - x;
    __syncthreads();
    if (threadIdx.x == blockDim.x - 1) carry = c + warp_sums[w] + incl;
    __syncthreads();
  }
}

// Stable scatter: the block walks its chunk in order, 256 elements at a time; ranks among equal
// digits come from __match_any_sync (within a warp) plus per-warp digit counts (across warps).
__global__ void __launch_bounds__(kRadixThreads) k_radix_scatter(
    int64_t N, int64_t chunk, int shift, const unsigned long long* __restrict__ kin,
    const uint32_t* __restrict__ vin, unsigned long long* __restrict__ kout,
    uint32_t* __restrict__ vout, const uint32_t* __restrict__ offs /* [bins][blocks] */) {
  constexpr int W = kRadixThreads / 32;
  __shared__ uint32_t s_off[kRadixBins];
  __shared__ uint32_t s_tot[kRadixBins];
  __shared__ uint32_t s_w[W][kRadixBins];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  for (int i = tid; i < kRadixBins; i += blockDim.x) {
    s_off[i] = offs[(int64_t)i * gridDim.x + blockIdx.x];
    for (int j = 0; j < W; ++j) s_w[j][i] = 0;
  }
  __syncthreads();
  const int64_t b0 = (int64_t)blockIdx.x * chunk, b1 = min(N, b0 + chunk);
  const unsigned lt = (1u << lane) - 1u;
  for (int64_t base = b0; base < b1; base += kRadixThreads) {
    const int64_t p = base + tid;
    const bool valid = p < b1;
    unsigned long long k = valid ? kin[p] : 0ull;
    uint32_t v = valid ? vin[p] : 0u;
    const int d = valid ? (int)((k >> shift) & (kRadixBins - 1)) : kRadixBins + lane;
    const unsigned peers = __match_any_sync(0xffffffffu, d);
    const int rank = __popc(peers & lt);
    if (valid && (__ffs(peers) - 1) == lane) s_w[w][d] = __popc(peers);
    __syncthreads();
    for (int i = tid; i < kRadixBins; i += blockDim.x) {
      uint32_t acc = 0;
      for (int j = 0; j < W; ++j) { uint32_t c = s_w[j][i]; s_w[j][i] = acc; acc += c; }
      s_tot[i] = acc;
    }
    __syncthreads();
    if (valid) {
      const uint32_t dst = s_off[d] + s_w[w][d] + rank;
      kout[dst] = k;
      vout[dst] = v;
    }
    __syncthreads();
    for (int i = tid; i < kRadixBins; i += blockDim.x) {
      s_off[i] += s_tot[i];
      for (int j = 0; j < W; ++j) s_w[j][i] = 0;
    }
    __syncthreads();
  }
}

__global__ void k_col_bounds(int64_t N, int m, const unsigned long long* __restrict__ keys,
                             int64_t* __restrict__ first, int64_t* __restrict__ last) {
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < N; p += (int64_t)gridDim.x * blockDim.x) {
    const int a = (int)(keys[p] >> 32);
    if (a >= m) continue;
    if (p == 0 || (int)(keys[p - 1] >> 32) != a) first[a] = p;
    if (p == N - 1 || (int)(keys[p + 1] >> 32) != a) last[a] = p + 1;
  }
}

__global__ void k_layout_scatter(int64_t N, int m, const unsigned long long* __restrict__ keys,
                                 const uint32_t* __restrict__ ids, const int64_t* __restrict__ first,
                                 const int64_t* __restrict__ col_start, float* __restrict__ val,
                                 int32_t* __restrict__ ins) {
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < N; p += (int64_t)gridDim.x * blockDim.x) {
    const unsigned long long k = keys[p];
    const int a = (int)(k >> 32);
    if (a >= m) continue;
    const uint32_t u = ~(uint32_t)k;  // fkey(v)
    const uint32_t b = (u & 0x80000000u) ? (u ^ 0x80000000u) : ~u;
    const int64_t dst = col_start[a] + (p - first[a]);
    val[dst] = __uint_as_float(b);
    ins[dst] = (int32_t)ids[p];
  }
}

// RLE: one run per maximal group of equal values inside an attribute list.  The lists are
// cut into PIECES of at most kRunPiece entries of one attribute (host-built, int4: attribute, first
// entry within the list, length, 0); one block per piece, so a few long attributes (C5: 18 lists of
// 5 M entries) use the whole GPU.  A run head is an entry whose value differs from its predecessor
// in the list (or the list's first entry).
constexpr int kRunPiece = 16384;

__device__ __forceinline__ bool run_head(const float* __restrict__ val, int64_t s, int64_t q) {
  return q == 0 || val[s + q] != val[s + q - 1];
}

// heads per piece (and per attribute)
__global__ void __launch_bounds__(256) k_run_heads(const int4* __restrict__ pieces, int np,
                                                   const int64_t* __restrict__ col_start,
                                                   const float* __restrict__ val, uint32_t* __restrict__ piece_cnt,
                                                   uint32_t* __restrict__ run_count) {
  __shared__ uint32_t ws[8];
  for (int pi = blockIdx.x; pi < np; pi += gridDim.x) {
    const int4 P = pieces[pi];
    const int64_t s = col_start[P.x];
    uint32_t c = 0;
    for (int64_t q = P.y + threadIdx.x; q < (int64_t)P.y + P.z; q += blockDim.x) c += run_head(val, s, q) ? 1u : 0u;
    for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = c;
    __syncthreads();
    if (threadIdx.x == 0) {
      uint32_t t = 0;
      for (int i = 0; i < 8; ++i) t += ws[i];
      piece_cnt[pi] = t;
      if (run_count) atomicAdd(run_count + P.x, t);
    }
    __syncthreads();
  }
}

// every head writes its run: value and list position (the run index = the piece's first run + the
// heads before it in the piece, by a block scan per 256-entry tile)
__global__ void __launch_bounds__(256) k_run_fill(const int4* __restrict__ pieces, int np,
                                                  const int64_t* __restrict__ col_start, const float* __restrict__ val,
                                                  const int64_t* __restrict__ piece_run, float* __restrict__ run_val,
                                                  int64_t* __restrict__ run_pos) {
  __shared__ uint32_t ws[8];
  __shared__ int64_t base_s;
  for (int pi = blockIdx.x; pi < np; pi += gridDim.x) {
    const int4 P = pieces[pi];
    const int64_t s = col_start[P.x];
    if (threadIdx.x == 0) base_s = piece_run[pi];
    __syncthreads();
    int64_t base = base_s;
    for (int64_t t0 = P.y; t0 < (int64_t)P.y + P.z; t0 += blockDim.x) {
      const int64_t q = t0 + threadIdx.x;
      const bool h = q < (int64_t)P.y + P.z && run_head(val, s, q);
      const unsigned bm = __ballot_sync(0xffffffffu, h);
      const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
      if (lane == 0) ws[w] = __popc(bm);
      __syncthreads();
      uint32_t before = 0, tot = 0;
      for (int i = 0; i < 8; ++i) { before += i < w ? ws[i] : 0u; tot += ws[i]; }
      if (h) {
        const int64_t r = base + before + __popc(bm & ((1u << lane) - 1u));
        run_val[r] = val[s + q];
        run_pos[r] = s + q;
      }
      base += tot;
      __syncthreads();
    }
  }
}

// run lengths from the positions; the segment -> run table of the root (one segment per
// attribute) and the run count
__global__ void k_run_pos(int m, const int64_t* __restrict__ col_start, const int64_t* __restrict__ col_len,
                          const int64_t* __restrict__ run_ptr, const int64_t* __restrict__ run_pos,
                          int32_t* __restrict__ run_len, int32_t* __restrict__ seg_run, int32_t* __restrict__ R) {
  const int64_t Rn = run_ptr[m];
  for (int a = blockIdx.x * blockDim.x + threadIdx.x; a <= m; a += gridDim.x * blockDim.x) {
    seg_run[a] = (int32_t)run_ptr[a];
    if (a == m) *R = (int32_t)Rn;
  }
  for (int64_t r = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; r < Rn; r += (int64_t)gridDim.x * blockDim.x) {
    int lo = 0, hi = m - 1;  // attribute of run r: the largest a with run_ptr[a] <= r
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (run_ptr[mid] <= r) lo = mid; else hi = mid - 1;
    }
    const int64_t end = r + 1 < run_ptr[lo + 1] ? run_pos[r + 1] : col_start[lo] + col_len[lo];
    run_len[r] = (int32_t)(end - run_pos[r]);
  }
}

// pieces of the lists of a shard (host)
static std::vector<int4> run_pieces(const Shard& sh) {
  std::vector<int4> pc;
  for (int a = 0; a < sh.m; ++a)
    for (int64_t o = 0; o < sh.h_col_len[(size_t)a]; o += kRunPiece)
      pc.push_back(make_int4(a, (int)o, (int)std::min<int64_t>(kRunPiece, sh.h_col_len[(size_t)a] - o), 0));
  return pc;
}

__global__ void k_run_chunk_root(int m, Tables tb) {
  const int R = *tb.R;
  for (int r = blockIdx.x * blockDim.x + threadIdx.x; r < R; r += gridDim.x * blockDim.x) {
    int lo = 0, hi = m - 1;  // attribute of run r
    while (lo < hi) { const int mid = (lo + hi + 1) >> 1; if (tb.seg_run[mid] <= r) lo = mid; else hi = mid - 1; }
    fill_run_chunks(tb.run_chunk, tb, lo, tb.run_pos[r], tb.run_len[r], r);
  }
}

// Present (non-NaN) entries per attribute: block-private shared-memory histograms when the
// attributes fit (one global add per attribute and block), plain global atomics otherwise.
constexpr int kHistSmem = 8192;
__global__ void k_col_hist(int64_t nnz, int64_t m, const int32_t* __restrict__ idx, const float* __restrict__ val,
                           unsigned long long* __restrict__ cnt) {
  __shared__ unsigned int hs[kHistSmem];
  const bool priv = m <= kHistSmem;
  if (priv)
    for (int a = threadIdx.x; a < m; a += blockDim.x) hs[a] = 0u;
  __syncthreads();
  for (int64_t p = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; p < nnz; p += (int64_t)gridDim.x * blockDim.x) {
    if (isnan(val[p])) continue;
    if (priv) atomicAdd(&hs[idx[p]], 1u);
    else atomicAdd(cnt + idx[p], 1ull);
  }
  if (priv) {
    __syncthreads();
    for (int a = threadIdx.x; a < m; a += blockDim.x)
      if (hs[a]) atomicAdd(cnt + a, (unsigned long long)hs[a]);
  }
}

}  // namespace

// Dense representation: the n x m matrix with every absent (or NaN)
// value filled with `fill` (the paper: "in the dense presentation, missing values need to be
// filled (e.g., treated as 0)"), as CSR rows of m entries each.  One thread per row.
__global__ void k_densify(int64_t n, int64_t m, const int64_t* __restrict__ indptr, const int32_t* __restrict__ idx,
                          const float* __restrict__ val, float fill, int64_t* __restrict__ dptr,
                          int32_t* __restrict__ didx, float* __restrict__ dval) {
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    float* row = dval + i * m;
    int32_t* ri = didx + i * m;
    for (int64_t a = 0; a < m; ++a) { row[a] = fill; ri[a] = (int32_t)a; }
    for (int64_t p = indptr[i]; p < indptr[i + 1]; ++p) {
      const int32_t a = idx[p];
      const float v = val[p];
      if (a < m && !isnan(v)) row[a] = v == 0.0f ? 0.0f : v;
    }
    dptr[i] = i * m;
    if (i == n - 1) dptr[n] = n * m;
  }
}

void densify(int64_t n, int64_t m, const int64_t* d_indptr, const int32_t* d_idx, const float* d_val, float fill,
             DBuf& optr, DBuf& oidx, DBuf& oval, cudaStream_t st) {
  optr.alloc((size_t)(n + 1) * 8, st);
  oidx.alloc((size_t)std::max<int64_t>(n * m, 1) * 4, st);
  oval.alloc((size_t)std::max<int64_t>(n * m, 1) * 4, st);
  const unsigned grid = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(n, 256), 148 * 8));
  k_densify<<<grid, 256, 0, st>>>(n, m, d_indptr, d_idx, d_val, fill, optr.as<int64_t>(), oidx.as<int32_t>(),
                                  oval.as<float>());
  GBDT_LAUNCH_CHECK();
}

// Runs (distinct values) of every attribute list of a built, uncompressed shard (AUTO RLE).
std::vector<uint32_t> attribute_runs(const Shard& sh, cudaStream_t st, int sms) {
  std::vector<uint32_t> hc((size_t)std::max(sh.m, 0), 0u);
  if (sh.m == 0 || sh.nnz == 0) return hc;
  const std::vector<int4> pc = run_pieces(sh);
  const int np = (int)pc.size();
  DBuf cnt((size_t)sh.m * 4, st), dpc((size_t)std::max(np, 1) * 16, st), pcnt((size_t)std::max(np, 1) * 4, st);
  GBDT_CUDA(cudaMemsetAsync(cnt.p, 0, (size_t)sh.m * 4, st));
  if (np) {
    GBDT_CUDA(cudaMemcpyAsync(dpc.p, pc.data(), (size_t)np * 16, cudaMemcpyHostToDevice, st));
    k_run_heads<<<(unsigned)std::min(np, sms * 16), 256, 0, st>>>(dpc.as<int4>(), np, sh.root.col_start,
                                                                 sh.val0.as<float>(), pcnt.as<uint32_t>(),
                                                                 cnt.as<uint32_t>());
    GBDT_LAUNCH_CHECK();
  }
  GBDT_CUDA(cudaMemcpyAsync(hc.data(), cnt.p, (size_t)sh.m * 4, cudaMemcpyDeviceToHost, st));
  GBDT_CUDA(cudaStreamSynchronize(st));
  return hc;
}

std::vector<int64_t> column_counts(int64_t nnz, int64_t m, const int32_t* d_indices, const float* d_values,
                                   cudaStream_t st) {
  int dev = 0, sms = 148;
  GBDT_CUDA(cudaGetDevice(&dev));
  GBDT_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev));
  DBuf c((size_t)m * 8, st);
  GBDT_CUDA(cudaMemsetAsync(c.p, 0, (size_t)m * 8, st));
  if (nnz > 0) {
    const unsigned g = (unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(nnz, 256), (int64_t)sms * 8));
    k_col_hist<<<g, 256, 0, st>>>(nnz, m, d_indices, d_values, c.as<unsigned long long>());
    GBDT_LAUNCH_CHECK();
  }
  std::vector<int64_t> h((size_t)m);
  GBDT_CUDA(cudaMemcpyAsync(h.data(), c.p, (size_t)m * 8, cudaMemcpyDeviceToHost, st));
  GBDT_CUDA(cudaStreamSynchronize(st));
  return h;
}

static void radix_sort(unsigned long long*& keys, uint32_t*& ids, unsigned long long*& kalt,
                       uint32_t*& ialt, int64_t N, int bits, cudaStream_t st, int sms) {
  if (N <= 1) return;
  const int64_t blocks = std::max<int64_t>(1, std::min<int64_t>(ceil_div(N, 8192), (int64_t)sms * 8));
  const int64_t chunk = ceil_div(ceil_div(N, blocks), kRadixThreads) * kRadixThreads;
  const int64_t nb = ceil_div(N, chunk);
  DBuf hist((size_t)kRadixBins * nb * sizeof(uint32_t), st);
  for (int shift = 0; shift < bits; shift += kRadixBits) {
    k_radix_hist<<<(unsigned)nb, kRadixThreads, 0, st>>>(N, chunk, shift, keys, hist.as<uint32_t>());
    GBDT_LAUNCH_CHECK();
    k_scan_u32<<<1, 1024, 0, st>>>((int64_t)kRadixBins * nb, hist.as<uint32_t>());
    GBDT_LAUNCH_CHECK();
    k_radix_scatter<<<(unsigned)nb, kRadixThreads, 0, st>>>(N, chunk, shift, keys, ids, kalt, ialt,
                                                            hist.as<uint32_t>());
    GBDT_LAUNCH_CHECK();
    std::swap(keys, kalt);
    std::swap(ids, ialt);
  }
}

void build_layout(Dataset& ds, const int64_t* d_indptr, const int32_t* d_indices,
                  const float* d_values, const std::vector<int64_t>& col_counts,
                  double rle_min_ratio) {
  cudaStream_t st = ds.stream;
  int sms = 148;
  GBDT_CUDA(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, ds.device));
  const int64_t N = ds.nnz;
  DBuf k0(std::max<int64_t>(N, 1) * 8, st), k1(std::max<int64_t>(N, 1) * 8, st);
  DBuf i0(std::max<int64_t>(N, 1) * 4, st), i1(std::max<int64_t>(N, 1) * 4, st);
  for (auto& shp : ds.shards) {
    Shard& sh = *shp;
    const int m = sh.m;
    // host-side column lengths (present entries; NaN counted out by the caller)
    sh.h_col_len.assign(m, 0);
    sh.nnz = 0;
    for (int a = 0; a < m; ++a) { sh.h_col_len[a] = col_counts[sh.a_begin + a]; sh.nnz += sh.h_col_len[a]; }
    sh.h_col_start.assign(m + 1, 0);
    std::vector<int32_t> tstart(m + 1, 0), cstart(m + 1, 0);
    for (int a = 0; a < m; ++a) {
      sh.h_col_start[a + 1] = sh.h_col_start[a] + pad4(sh.h_col_len[a]);
      tstart[a + 1] = tstart[a] + (int32_t)ceil_div(sh.h_col_len[a], kTile);
      cstart[a + 1] = cstart[a] + (int32_t)ceil_div(sh.h_col_len[a], kChunk);
    }
    sh.T0 = tstart[m];
    sh.C0 = cstart[m];
    sh.cap = sh.h_col_start[m] + 16;
    sh.val0.alloc(sh.cap * 4, st);
    sh.ins0.alloc(sh.cap * 4, st);
    GBDT_CUDA(cudaMemsetAsync(sh.val0.p, 0, sh.cap * 4, st));
    GBDT_CUDA(cudaMemsetAsync(sh.ins0.p, 0, sh.cap * 4, st));
    for (int b = 0; b < 2; ++b) {
      sh.valw[b].alloc(sh.cap * 4, st);
      sh.insw[b].alloc(sh.cap * 4, st);
      GBDT_CUDA(cudaMemsetAsync(sh.valw[b].p, 0, sh.cap * 4, st));
      GBDT_CUDA(cudaMemsetAsync(sh.insw[b].p, 0, sh.cap * 4, st));
    }
    // root tables: col_start[m+1], col_len[m], tile_start[m+1], seg_start[m], seg_cnt[m], T
    const size_t rb = (size_t)(m + 1) * 8 + (size_t)m * 8 + (size_t)(m + 1) * 8 + (size_t)m * 16 + 64;
    sh.root_tab.alloc(rb + 64, st);
    char* q = sh.root_tab.as<char>();
    sh.root.col_start = (int64_t*)q; q += (size_t)(m + 1) * 8;
    sh.root.col_len = (int64_t*)q; q += (size_t)m * 8;
    sh.root.seg_start = (int64_t*)q; q += (size_t)m * 8;
    sh.root.seg_cnt = (int64_t*)q; q += (size_t)m * 8;
    sh.root.T = (int32_t*)q; q += 16;
    sh.root.C = (int32_t*)q; q += 16;
    sh.root.tile_start = (int32_t*)q; q += (size_t)(m + 1) * 4;
    sh.root.chunk_start = (int32_t*)q;
    GBDT_CUDA(cudaMemcpyAsync(sh.root.col_start, sh.h_col_start.data(), (m + 1) * 8, cudaMemcpyHostToDevice, st));
    if (m) {
      GBDT_CUDA(cudaMemcpyAsync(sh.root.col_len, sh.h_col_len.data(), m * 8, cudaMemcpyHostToDevice, st));
      GBDT_CUDA(cudaMemcpyAsync(sh.root.seg_start, sh.h_col_start.data(), m * 8, cudaMemcpyHostToDevice, st));
      GBDT_CUDA(cudaMemcpyAsync(sh.root.seg_cnt, sh.h_col_len.data(), m * 8, cudaMemcpyHostToDevice, st));
    }
    GBDT_CUDA(cudaMemcpyAsync(sh.root.tile_start, tstart.data(), (m + 1) * 4, cudaMemcpyHostToDevice, st));
    GBDT_CUDA(cudaMemcpyAsync(sh.root.T, &sh.T0, 4, cudaMemcpyHostToDevice, st));
    GBDT_CUDA(cudaMemcpyAsync(sh.root.chunk_start, cstart.data(), (m + 1) * 4, cudaMemcpyHostToDevice, st));
    GBDT_CUDA(cudaMemcpyAsync(sh.root.C, &sh.C0, 4, cudaMemcpyHostToDevice, st));
    std::vector<int32_t> cattr((size_t)std::max(sh.C0, 1), 0);
    for (int a = 0; a < m; ++a)
      for (int c = cstart[a]; c < cstart[a + 1]; ++c) cattr[c] = a;
    sh.root_chunk_attr.alloc(cattr.size() * 4, st);
    sh.root.chunk_attr = sh.root_chunk_attr.as<int32_t>();
    GBDT_CUDA(cudaMemcpyAsync(sh.root.chunk_attr, cattr.data(), cattr.size() * 4, cudaMemcpyHostToDevice, st));
    GBDT_CUDA(cudaStreamSynchronize(st));  // host vectors above must outlive the copies
    if (m == 0 || sh.nnz == 0) continue;

    unsigned long long* keys = k0.as<unsigned long long>();
    unsigned long long* kalt = k1.as<unsigned long long>();
    uint32_t* ids = i0.as<uint32_t>();
    uint32_t* ialt = i1.as<uint32_t>();
    k_make_keys<<<(unsigned)std::min<int64_t>(ceil_div(ds.n, 8), (int64_t)sms * 32), 256, 0, st>>>(
        ds.n, d_indptr, d_indices, d_values, sh.a_begin, sh.a_end, keys, ids);
    GBDT_LAUNCH_CHECK();
    int abits = 1;
    while ((1ll << abits) <= m) ++abits;  // room for the sentinel value m
    radix_sort(keys, ids, kalt, ialt, N, 32 + abits, st, sms);
    DBuf first((size_t)m * 8, st), last((size_t)m * 8, st);
    GBDT_CUDA(cudaMemsetAsync(first.p, 0, (size_t)m * 8, st));
    GBDT_CUDA(cudaMemsetAsync(last.p, 0, (size_t)m * 8, st));
    const unsigned g = (unsigned)std::min<int64_t>(ceil_div(N, 256), (int64_t)sms * 16);
    k_col_bounds<<<g, 256, 0, st>>>(N, m, keys, first.as<int64_t>(), last.as<int64_t>());
    GBDT_LAUNCH_CHECK();
    k_layout_scatter<<<g, 256, 0, st>>>(N, m, keys, ids, first.as<int64_t>(), sh.root.col_start,
                                        sh.val0.as<float>(), sh.ins0.as<int32_t>());
    GBDT_LAUNCH_CHECK();

    // ---- optional RLE of the sorted lists
    if (ds.rle != GBDT_RLE_OFF) {
      const std::vector<int4> pc = run_pieces(sh);
      const int np = (int)pc.size();
      DBuf cnt((size_t)m * 4, st), dpc((size_t)std::max(np, 1) * 16, st), pcnt((size_t)std::max(np, 1) * 4, st);
      GBDT_CUDA(cudaMemsetAsync(cnt.p, 0, (size_t)m * 4, st));
      if (np) {
        GBDT_CUDA(cudaMemcpyAsync(dpc.p, pc.data(), (size_t)np * 16, cudaMemcpyHostToDevice, st));
        k_run_heads<<<(unsigned)std::min(np, sms * 16), 256, 0, st>>>(dpc.as<int4>(), np, sh.root.col_start,
                                                                     sh.val0.as<float>(), pcnt.as<uint32_t>(),
                                                                     cnt.as<uint32_t>());
        GBDT_LAUNCH_CHECK();
      }
      std::vector<uint32_t> hc(m), hp((size_t)np);
      GBDT_CUDA(cudaMemcpyAsync(hc.data(), cnt.p, (size_t)m * 4, cudaMemcpyDeviceToHost, st));
      if (np) GBDT_CUDA(cudaMemcpyAsync(hp.data(), pcnt.p, (size_t)np * 4, cudaMemcpyDeviceToHost, st));
      GBDT_CUDA(cudaStreamSynchronize(st));
      int64_t R = 0, entries = 0;
      for (int a = 0; a < m; ++a) { R += hc[a]; entries += sh.h_col_len[a]; }
      const double ratio = R ? (double)entries / (double)R : 0.0;
      const double thr = rle_min_ratio > 0 ? rle_min_ratio : 2.0;
      if (ds.rle == GBDT_RLE_ON || ratio >= thr) {
        std::vector<int64_t> rp(m + 1, 0);
        for (int a = 0; a < m; ++a) rp[a + 1] = rp[a] + hc[a];
        std::vector<int64_t> prun((size_t)std::max(np, 1), 0);  // first run of every piece
        {
          int64_t acc = 0;
          for (int i = 0; i < np; ++i) { prun[(size_t)i] = acc; acc += hp[(size_t)i]; }
        }
        sh.rle = true;
        sh.runs = R;
        sh.run_ptr.alloc((size_t)(m + 1) * 8, st);
        sh.run_val.alloc((size_t)std::max<int64_t>(R, 1) * 4 + 64, st);
        sh.run_len.alloc((size_t)std::max<int64_t>(R, 1) * 4 + 64, st);
        sh.run_pos.alloc((size_t)std::max<int64_t>(R, 1) * 8 + 64, st);
        DBuf dprun((size_t)std::max(np, 1) * 8, st);
        GBDT_CUDA(cudaMemcpyAsync(sh.run_ptr.p, rp.data(), (size_t)(m + 1) * 8, cudaMemcpyHostToDevice, st));
        if (np) {
          GBDT_CUDA(cudaMemcpyAsync(dprun.p, prun.data(), (size_t)np * 8, cudaMemcpyHostToDevice, st));
          k_run_fill<<<(unsigned)std::min(np, sms * 16), 256, 0, st>>>(dpc.as<int4>(), np, sh.root.col_start,
                                                                      sh.val0.as<float>(), dprun.as<int64_t>(),
                                                                      sh.run_val.as<float>(), sh.run_pos.as<int64_t>());
          GBDT_LAUNCH_CHECK();
        }
        sh.run_seg.alloc((size_t)(m + 1) * 4 + 64, st);
        int32_t* Rdev = reinterpret_cast<int32_t*>(sh.run_seg.as<char>() + (size_t)(m + 1) * 4 + 16);
        k_run_pos<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(std::max<int64_t>(R, m + 1), 256), (int64_t)sms * 8)), 256, 0, st>>>(
            m, sh.root.col_start, sh.root.col_len, sh.run_ptr.as<int64_t>(), sh.run_pos.as<int64_t>(),
            sh.run_len.as<int32_t>(), sh.run_seg.as<int32_t>(), Rdev);
        GBDT_LAUNCH_CHECK();
        GBDT_CUDA(cudaStreamSynchronize(st));  // the host vectors (pieces, piece runs) outlive the copies
        sh.root.seg_run = sh.run_seg.as<int32_t>();
        sh.root.run_val = sh.run_val.as<float>();
        sh.root.run_len = sh.run_len.as<int32_t>();
        sh.root.run_pos = sh.run_pos.as<int64_t>();
        sh.root.R = Rdev;
        sh.run_chunk.alloc((size_t)std::max(sh.C0, 1) * 4 + 64, st);
        sh.root.run_chunk = sh.run_chunk.as<int32_t>();
        k_run_chunk_root<<<(unsigned)std::max<int64_t>(1, std::min<int64_t>(ceil_div(R, 256), (int64_t)sms * 8)), 256, 0, st>>>(
            m, sh.root);
        GBDT_LAUNCH_CHECK();
        GBDT_CUDA(cudaStreamSynchronize(st));
      }
    }
  }
  GBDT_CUDA(cudaStreamSynchronize(ds.stream));
}

}  // namespace gbdt
