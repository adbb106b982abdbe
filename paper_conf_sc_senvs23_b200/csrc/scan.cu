// scan.cu — device-wide exclusive scan of u32 counts (site / chain-pool compaction, SURVEY a-7).
// Three phases: per-tile sums, one CTA scans the tile sums, per-tile rescan + offset.
#include <cuda_runtime.h>

#include "ctx.h"

namespace gs {
namespace {

constexpr int kThreads = 1024, kItems = 4, kTile = kThreads * kItems;

__device__ __forceinline__ unsigned long long warp_incl(unsigned long long v) {
  const int lane = threadIdx.x & 31;
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long x = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += x;
  }
  return v;
}
// exclusive block scan of one value per thread; returns the exclusive prefix, *total = block sum
__device__ unsigned long long block_excl(unsigned long long v, unsigned long long* total) {
  __shared__ unsigned long long ws[kThreads / 32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const unsigned long long inc = warp_incl(v);
  if (lane == 31) ws[warp] = inc;
  __syncthreads();
  if (warp == 0) {
    unsigned long long x = lane < kThreads / 32 ? ws[lane] : 0;
    x = warp_incl(x);
    if (lane < kThreads / 32) ws[lane] = x;
  }
  __syncthreads();
  const unsigned long long before = warp ? ws[warp - 1] : 0;
  *total = ws[kThreads / 32 - 1];
  __syncthreads();
  return before + inc - v;
}

__global__ void __launch_bounds__(kThreads) k_tile_sum(const uint32_t* __restrict__ in, uint64_t n,
                                                       unsigned long long* __restrict__ bsum) {
  const uint64_t base = (uint64_t)blockIdx.x * kTile + (uint64_t)threadIdx.x * kItems;
  unsigned long long s = 0;
#pragma unroll
  for (int q = 0; q < kItems; q++) s += base + q < n ? in[base + q] : 0u;
  unsigned long long tot;
  block_excl(s, &tot);
  if (threadIdx.x == 0) bsum[blockIdx.x] = tot;
}

__global__ void __launch_bounds__(kThreads) k_scan_bsum(unsigned long long* bsum, uint64_t nb,
                                                        unsigned long long* d_total) {
  unsigned long long carry = 0;
  for (uint64_t b = 0; b < nb; b += kThreads) {
    const uint64_t i = b + threadIdx.x;
    const unsigned long long v = i < nb ? bsum[i] : 0;
    unsigned long long tot;
    const unsigned long long ex = block_excl(v, &tot);
    if (i < nb) bsum[i] = carry + ex;
    carry += tot;
  }
  if (threadIdx.x == 0) *d_total = carry;
}

template <typename OutT>
__global__ void __launch_bounds__(kThreads) k_tile_apply(const uint32_t* __restrict__ in, uint64_t n,
                                                         const unsigned long long* __restrict__ bsum,
                                                         OutT* __restrict__ out) {
  const uint64_t base = (uint64_t)blockIdx.x * kTile + (uint64_t)threadIdx.x * kItems;
  uint32_t v[kItems];
  unsigned long long s = 0;
#pragma unroll
  for (int q = 0; q < kItems; q++) {
    v[q] = base + q < n ? in[base + q] : 0u;
    s += v[q];
  }
  unsigned long long tot;
  unsigned long long ex = block_excl(s, &tot) + bsum[blockIdx.x];
#pragma unroll
  for (int q = 0; q < kItems; q++) {
    if (base + q < n) out[base + q] = (OutT)ex;
    ex += v[q];
  }
}

template <typename OutT>
gs_status scan_impl(gs_ctx* c, const uint32_t* in, OutT* out, uint64_t n, unsigned long long* d_total) {
  const uint64_t nb = (n + kTile - 1) / kTile;
  const size_t need = (nb ? nb : 1) * sizeof(unsigned long long);
  if (c->scan_tmp_bytes < need) {
    if (c->d_scan_tmp) cudaFree(c->d_scan_tmp);
    c->d_scan_tmp = nullptr;
    c->scan_tmp_bytes = 0;
    GS_CUDA(c, cudaMalloc(&c->d_scan_tmp, need));
    c->scan_tmp_bytes = need;
  }
  unsigned long long* bs = static_cast<unsigned long long*>(c->d_scan_tmp);
  if (nb == 0) {
    GS_CUDA(c, cudaMemsetAsync(d_total, 0, 8, c->stream));
    return GS_OK;
  }
  k_tile_sum<<<(unsigned)nb, kThreads, 0, c->stream>>>(in, n, bs); count_launch();
  k_scan_bsum<<<1, kThreads, 0, c->stream>>>(bs, nb, d_total); count_launch();
  k_tile_apply<OutT><<<(unsigned)nb, kThreads, 0, c->stream>>>(in, n, bs, out); count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

}  // namespace

gs_status scan_u32(gs_ctx* c, const uint32_t* in, uint32_t* out, uint64_t n, unsigned long long* d_total) {
  return scan_impl<uint32_t>(c, in, out, n, d_total);
}
gs_status scan_u32_to_u64(gs_ctx* c, const uint32_t* in, unsigned long long* out, uint64_t n,
                          unsigned long long* d_total) {
  return scan_impl<unsigned long long>(c, in, out, n, d_total);
}

}  // namespace gs
