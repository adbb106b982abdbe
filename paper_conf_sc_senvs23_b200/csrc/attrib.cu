// attrib.cu — PC-sample packing and the per-PC x stall-reason histogram
// (§2.2, §3).
//
// Packed sample word: (slot << 5) | reason, slot = first_slot[kernel] + pc/16 (R30). Because a
// histogram row is 32 bins wide the word IS the flat bin index, so the hot loop is
// "validate, then increment H[word]". Strategies (gs_config.hist_mode):
//   PRIVATE  the compact bin space (slot * n_reasons + reason) is split into ranges that fit one
//            CTA's shared memory; each CTA streams a contiguous chunk of samples with 128-bit
//            loads and counts the samples of its range with shared-memory atomics; the CTAs of
//            one chunk are launched adjacently so the repeated reads of a chunk hit L2. Counts
//            are flushed to the global histogram once per CTA.
//   GLOBAL   one L2 atomic (RED) per valid sample.
//   AUTO     PRIVATE when the compact bin space needs at most kMaxRanges ranges, else GLOBAL.
#include <cuda_runtime.h>

#include <algorithm>

#include "ctx.h"

namespace gs {
namespace {

constexpr int kThreads = 512;
constexpr uint32_t kRangeBins = 48 * 1024;  // u32 counters per CTA (192 KB of shared memory)
constexpr uint32_t kMaxRanges = 8;

__device__ __forceinline__ void count_invalid(uint32_t n_bad, unsigned long long* d_n_invalid) {
  // n_bad per thread -> one atomic per warp
  for (int o = 16; o; o >>= 1) n_bad += __shfl_xor_sync(0xffffffffu, n_bad, o);
  if ((threadIdx.x & 31) == 0 && n_bad) atomicAdd(d_n_invalid, (unsigned long long)n_bad);
}

__global__ void k_pack(const uint32_t* __restrict__ raw, uint64_t n, const KDesc* __restrict__ kd, uint32_t nk,
                       uint32_t nr, uint32_t* __restrict__ words, unsigned long long* d_n_invalid) {
  const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  uint32_t bad = 0;
  if (i < n) {
    const uint32_t k = raw[3 * i], pc = raw[3 * i + 1], reason = raw[3 * i + 2];
    bool ok = k < nk && (pc & 15u) == 0 && reason < nr;
    uint32_t w = 0xffffffffu;
    if (ok) {
      const KDesc K = kd[k];
      ok = (pc >> 4) < K.n;
      if (ok) w = ((K.first + (pc >> 4)) << 5) | reason;
    }
    words[i] = w;
    bad = ok ? 0 : 1;
  }
  count_invalid(bad, d_n_invalid);
}

// -------------------------------------------------------------------------------- GLOBAL
__global__ void __launch_bounds__(kThreads) k_hist_global(const uint32_t* __restrict__ s, uint64_t n, uint32_t P,
                                                          uint32_t nr, int32_t* __restrict__ H,
                                                          unsigned long long* d_n_invalid) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  uint32_t bad = 0;
  const uint64_t n4 = n / 4;
  const uint4* s4 = reinterpret_cast<const uint4*>(s);
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n4; i += stride) {
    const uint4 v = __ldg(s4 + i);
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int q = 0; q < 4; q++) {
      if ((w[q] >> 5) < P && (w[q] & 31u) < nr) atomicAdd(H + w[q], 1);
      else bad++;
    }
  }
  for (uint64_t i = n4 * 4 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
    const uint32_t w = s[i];
    if ((w >> 5) < P && (w & 31u) < nr) atomicAdd(H + w, 1);
    else bad++;
  }
  count_invalid(bad, d_n_invalid);
}

// -------------------------------------------------------------------------------- PRIVATE
// grid = n_chunks * n_ranges; blockIdx.x = chunk * n_ranges + range
__global__ void __launch_bounds__(kThreads) k_hist_private(const uint32_t* __restrict__ s, uint64_t n, uint32_t P,
                                                           uint32_t nr, uint32_t n_ranges, uint32_t range_bins,
                                                           uint64_t chunk, int32_t* __restrict__ H,
                                                           unsigned long long* d_n_invalid) {
  extern __shared__ uint32_t cnt[];
  const uint32_t range = blockIdx.x % n_ranges;
  const uint64_t ci = blockIdx.x / n_ranges;
  const uint32_t lo = range * range_bins;
  for (uint32_t b = threadIdx.x; b < range_bins; b += blockDim.x) cnt[b] = 0;
  __syncthreads();
  uint64_t a = ci * chunk, e = a + chunk;
  if (e > n) e = n;
  uint32_t bad = 0;
  // chunk starts are multiples of 4 words: 128-bit loads for the body
  const uint64_t a4 = a / 4, e4 = e / 4;
  const uint4* s4 = reinterpret_cast<const uint4*>(s);
  for (uint64_t i = a4 + threadIdx.x; i < e4; i += blockDim.x) {
    const uint4 v = __ldg(s4 + i);
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int q = 0; q < 4; q++) {
      const uint32_t slot = w[q] >> 5, rs = w[q] & 31u;
      if (slot < P && rs < nr) {
        const uint32_t cb = slot * nr + rs - lo;
        if (cb < range_bins) atomicAdd(cnt + cb, 1u);
      } else {
        bad++;
      }
    }
  }
  for (uint64_t i = e4 * 4 + threadIdx.x; i < e; i += blockDim.x) {
    const uint32_t w = s[i], slot = w >> 5, rs = w & 31u;
    if (slot < P && rs < nr) {
      const uint32_t cb = slot * nr + rs - lo;
      if (cb < range_bins) atomicAdd(cnt + cb, 1u);
    } else {
      bad++;
    }
  }
  if (range == 0) count_invalid(bad, d_n_invalid);
  __syncthreads();
  for (uint32_t b = threadIdx.x; b < range_bins; b += blockDim.x) {
    const uint32_t v = cnt[b];
    if (v) {
      const uint32_t cbg = lo + b;
      atomicAdd(H + (cbg / nr) * 32u + cbg % nr, (int32_t)v);
    }
  }
}

}  // namespace

gs_status pack_samples_run(gs_ctx* c, const uint32_t* d_raw, uint64_t n, uint32_t* d_words,
                           unsigned long long* d_n_invalid) {
  if (!n) return GS_OK;
  k_pack<<<(unsigned)((n + 255) / 256), 256, 0, c->stream>>>(d_raw, n, c->d_kd, c->n_kernels, c->cfg.n_reasons,
                                                             d_words, d_n_invalid); count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

gs_status hist_run(gs_ctx* c, const uint32_t* d_words, uint64_t n, int32_t* d_hist, unsigned long long* d_n_invalid,
                   int accumulate, bool zero_first) {
  cudaStream_t st = c->stream;
  const uint32_t P = (uint32_t)c->n_instr, nr = c->cfg.n_reasons;
  if (zero_first && !accumulate) GS_CUDA(c, cudaMemsetAsync(d_hist, 0, (uint64_t)P * 32 * 4, st));
  if (!n) return GS_OK;
  int dev_sms = 148;
  cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, c->device);
  const uint64_t compact = (uint64_t)P * nr;
  uint32_t mode = c->cfg.hist_mode;
  const uint32_t n_ranges = (uint32_t)((compact + kRangeBins - 1) / kRangeBins);
  if (reinterpret_cast<uintptr_t>(d_words) & 3u) return fail(c, GS_E_INVAL, "sample pointer must be 4-byte aligned");
  // peel the words before the first 16-byte boundary so the main kernels use 128-bit loads
  const uint64_t head = std::min<uint64_t>(n, ((16u - (reinterpret_cast<uintptr_t>(d_words) & 15u)) & 15u) / 4u);
  if (head) {
    k_hist_global<<<1, 32, 0, st>>>(d_words, head, P, nr, d_hist, d_n_invalid); count_launch();
    GS_CUDA(c, cudaGetLastError());
    d_words += head;
    n -= head;
    if (!n) return GS_OK;
  }
  if (mode == GS_HIST_AUTO) mode = (n_ranges <= kMaxRanges) ? GS_HIST_PRIVATE : GS_HIST_GLOBAL;
  if (mode == GS_HIST_PRIVATE && n_ranges > 64) mode = GS_HIST_GLOBAL;
  if (mode == GS_HIST_WINDOW) mode = GS_HIST_GLOBAL;  // not implemented yet
  c->last_hist_mode = (int)mode;
  if (mode == GS_HIST_GLOBAL) {
    const uint64_t blocks = std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)dev_sms * 4, (n + kThreads * 4 - 1) / (kThreads * 4)));
    k_hist_global<<<(unsigned)blocks, kThreads, 0, st>>>(d_words, n, P, nr, d_hist, d_n_invalid); count_launch();
    GS_CUDA(c, cudaGetLastError());
    return GS_OK;
  }
  // PRIVATE: bins per range, chunk size so that every CTA sees >= 4 samples per bin of its range
  const uint32_t range_bins = (uint32_t)((compact + n_ranges - 1) / n_ranges);
  const size_t smem = (size_t)range_bins * 4;
  GS_CUDA(c, cudaFuncSetAttribute(k_hist_private, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  int per_sm = 1;
  GS_CUDA(c, cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, k_hist_private, kThreads, smem));
  per_sm = std::max(per_sm, 1);
  uint64_t chunks = std::max<uint64_t>(1, ((uint64_t)dev_sms * per_sm) / n_ranges);
  chunks = std::min<uint64_t>(chunks, std::max<uint64_t>(1, n / (4ull * range_bins)));
  uint64_t chunk = (n + chunks - 1) / chunks;
  chunk = (chunk + 3) & ~3ull;
  chunks = (n + chunk - 1) / chunk;
  k_hist_private<<<(unsigned)(chunks * n_ranges), kThreads, smem, st>>>(d_words, n, P, nr, n_ranges, range_bins, chunk,
                                                                       d_hist, d_n_invalid); count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

void attrib_free(gs_ctx* c) {
  for (int b = 0; b < 2; b++) {
    if (c->h_stage[b]) cudaFreeHost(c->h_stage[b]);
    if (c->d_stage[b]) cudaFree(c->d_stage[b]);
    if (c->ev_stage[b]) cudaEventDestroy(c->ev_stage[b]);
    c->h_stage[b] = nullptr;
    c->d_stage[b] = nullptr;
    c->ev_stage[b] = nullptr;
  }
  c->stage_words = 0;
}

}  // namespace gs
