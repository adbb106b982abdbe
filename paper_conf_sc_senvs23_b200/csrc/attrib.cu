// attrib.cu — PC-sample packing and the per-PC x stall-reason histogram
// (§2.2, §3).
//
// Packed sample word: (slot << 5) | reason, slot = first_slot[kernel] + pc/16 (R30). Because a
// histogram row is 32 bins wide the word IS the flat bin index: the hot loop is "validate, then
// increment H[word]". Global atomics alone run at ~50-200 G samples/s on B200 (L2 atomic rate,
// profiles/r01_atomics_microbench.txt) — far below the ~1.6 T samples/s HBM streams 4-byte
// samples at — so the counting happens in shared memory:
//
//   * compact bins cb = slot * n_reasons + reason (only active reasons occupy shared memory);
//   * the table packs two 16-bit counters per 32-bit word (114688 bins in 224 KB, one CTA
//     of 1024 threads per SM); a counter that reaches 0x8000 is drained (-0x8000 in shared
//     memory, +0x8000 to the global bin) by the one thread whose atomicAdd returned 0x7FFF, so a
//     16-bit half can never carry into its neighbour (at most a few thousand increments can be in
//     flight per SM between that add and the drain) and the counts stay exact;
//   * samples stream in with 128-bit loads.
// Strategies (gs_config.hist_mode):
//   PRIVATE  fixed windows: the compact bin space is split into ranges of one table each; each
//            CTA counts the samples of its range in a contiguous chunk; the CTAs of one chunk are
//            launched adjacently so the re-reads of a chunk hit L2. Flushed once per CTA.
//   WINDOW   one persistent CTA per SM streams a contiguous 1/grid of the samples in tiles and
//            moves its window with the data: at a tile whose first sample falls outside the
//            window, the table is flushed and re-based at the sample's kernel (whole kernel if it
//            fits, else centred on the sample). Samples outside the window go straight to L2
//            atomics. Suited to PC-sampling traces, which arrive grouped by kernel launch.
//   GLOBAL   one L2 atomic per valid sample (reference strategy).
//   AUTO     PRIVATE if the compact bins fit in kMaxRanges tables, else WINDOW.
#include <cuda_runtime.h>

#include <algorithm>

#include "ctx.h"

namespace gs {
namespace {

constexpr int kThreadsGlobal = 512;
constexpr int kThreadsSmem = 1024;
constexpr uint32_t kTableWords = 56 * 1024;        // 224 KB of shared memory
constexpr uint32_t kTableBins = 2 * kTableWords;   // 114688 16-bit counters
constexpr uint32_t kMaxRanges = 3;
constexpr uint32_t kTile4 = 8192;                  // uint4 per window decision (32K samples)
constexpr uint32_t kNoWindow = 0xffffffffu;

__device__ __forceinline__ void count_invalid(uint32_t n_bad, unsigned long long* d_n_invalid) {
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
__global__ void __launch_bounds__(kThreadsGlobal) k_hist_global(const uint32_t* __restrict__ s, uint64_t n, uint32_t P,
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

// -------------------------------------------------------------------------------- shared-memory table
__device__ __forceinline__ uint32_t word_of(uint32_t cb, uint32_t nr) { return (cb / nr) * 32u + cb % nr; }

// one sample: shared-memory 16-bit counter if inside the window; outside it an L2 atomic (WINDOW)
// or nothing (PRIVATE: another CTA owns that range)
template <bool SPILL_OUT>
__device__ __forceinline__ void count_one(uint32_t w, uint32_t P, uint32_t nr, uint32_t wb, uint32_t* tab,
                                          int32_t* H, uint32_t& bad) {
  const uint32_t slot = w >> 5, rs = w & 31u;
  if (slot < P && rs < nr) {
    const uint32_t off = slot * nr + rs - wb;
    if (off < kTableBins) {
      const uint32_t sh = (off & 1u) << 4;
      const uint32_t old = atomicAdd(tab + (off >> 1), 1u << sh);
      if (((old >> sh) & 0xffffu) == 0x7fffu) {  // drain: keep every 16-bit half below 2^16
        atomicSub(tab + (off >> 1), 0x8000u << sh);
        atomicAdd(H + w, 0x8000);
      }
    } else if (SPILL_OUT) {
      atomicAdd(H + w, 1);
    }
  } else {
    bad++;
  }
}

__device__ void flush_table(uint32_t* tab, uint32_t wb, uint32_t nr, int32_t* H) {
  for (uint32_t i = threadIdx.x; i < kTableWords; i += blockDim.x) {
    const uint32_t v = tab[i];
    if (!v) continue;
    tab[i] = 0;
    const uint32_t cb = wb + 2 * i;
    if (v & 0xffffu) atomicAdd(H + word_of(cb, nr), (int32_t)(v & 0xffffu));
    if (v >> 16) atomicAdd(H + word_of(cb + 1, nr), (int32_t)(v >> 16));
  }
}

// DYN = false: PRIVATE (fixed range per CTA); DYN = true: WINDOW (window follows the data)
template <bool DYN>
__global__ void __launch_bounds__(kThreadsSmem, 1)
    k_hist_smem(const uint32_t* __restrict__ s, uint64_t n, uint32_t P, uint32_t nr, const KDesc* __restrict__ kd,
                uint32_t nk, uint32_t n_ranges, uint64_t chunk, int32_t* __restrict__ H,
                unsigned long long* d_n_invalid) {
  extern __shared__ uint32_t tab[];
  __shared__ uint32_t sh_wb[2];
  const uint32_t range = DYN ? 0u : blockIdx.x % n_ranges;
  const uint64_t ci = DYN ? blockIdx.x : blockIdx.x / n_ranges;
  uint32_t wb = DYN ? kNoWindow : range * kTableBins;
  for (uint32_t i = threadIdx.x; i < kTableWords; i += blockDim.x) tab[i] = 0;
  const uint64_t a = ci * chunk;
  const uint64_t e = a + chunk < n ? a + chunk : n;
  uint32_t bad = 0;
  const uint4* s4 = reinterpret_cast<const uint4*>(s);
  const uint64_t a4 = a / 4, e4 = e / 4;
  __syncthreads();
  uint32_t it = 0;
  for (uint64_t t4 = a4; t4 < e4; t4 += kTile4, it++) {
    const uint64_t t4e = t4 + kTile4 < e4 ? t4 + kTile4 : e4;
    if (DYN) {
      if (threadIdx.x == 0) {
        uint32_t nwb = wb;
        const uint32_t w = s[4 * t4], slot = w >> 5, rs = w & 31u;
        if (slot < P && rs < nr) {
          const uint32_t cb = slot * nr + rs;
          if (wb == kNoWindow || cb - wb >= kTableBins) {
            uint32_t lo = 0, hi = nk;  // kernel of the slot: last k with first <= slot
            while (hi - lo > 1) {
              const uint32_t mid = (lo + hi) >> 1;
              if (kd[mid].first <= slot) lo = mid;
              else hi = mid;
            }
            const uint32_t kb0 = kd[lo].first * nr, kbins = kd[lo].n * nr;
            nwb = kbins <= kTableBins ? kb0 : (cb > kTableBins / 2 ? cb - kTableBins / 2 : 0);
          }
        }
        if (nwb == kNoWindow) nwb = 0;  // first tile starts with an invalid sample
        sh_wb[it & 1] = nwb;
      }
      __syncthreads();
      const uint32_t nwb = sh_wb[it & 1];
      if (nwb != wb) {
        if (wb != kNoWindow) {
          flush_table(tab, wb, nr, H);
          __syncthreads();
        }
        wb = nwb;
      }
    }
    uint64_t i = t4 + threadIdx.x;
    for (; i + blockDim.x < t4e; i += 2 * blockDim.x) {  // two 128-bit loads in flight per thread
      const uint4 v0 = __ldg(s4 + i), v1 = __ldg(s4 + i + blockDim.x);
      count_one<DYN>(v0.x, P, nr, wb, tab, H, bad);
      count_one<DYN>(v0.y, P, nr, wb, tab, H, bad);
      count_one<DYN>(v0.z, P, nr, wb, tab, H, bad);
      count_one<DYN>(v0.w, P, nr, wb, tab, H, bad);
      count_one<DYN>(v1.x, P, nr, wb, tab, H, bad);
      count_one<DYN>(v1.y, P, nr, wb, tab, H, bad);
      count_one<DYN>(v1.z, P, nr, wb, tab, H, bad);
      count_one<DYN>(v1.w, P, nr, wb, tab, H, bad);
    }
    if (i < t4e) {
      const uint4 v0 = __ldg(s4 + i);
      count_one<DYN>(v0.x, P, nr, wb, tab, H, bad);
      count_one<DYN>(v0.y, P, nr, wb, tab, H, bad);
      count_one<DYN>(v0.z, P, nr, wb, tab, H, bad);
      count_one<DYN>(v0.w, P, nr, wb, tab, H, bad);
    }
  }
  for (uint64_t i = e4 * 4 + threadIdx.x; i < e; i += blockDim.x) count_one<DYN>(s[i], P, nr, wb, tab, H, bad);
  if (range == 0) count_invalid(bad, d_n_invalid);
  __syncthreads();
  if (wb != kNoWindow) flush_table(tab, wb, nr, H);
}

}  // namespace

gs_status pack_samples_run(gs_ctx* c, const uint32_t* d_raw, uint64_t n, uint32_t* d_words,
                           unsigned long long* d_n_invalid) {
  if (!n) return GS_OK;
  k_pack<<<(unsigned)((n + 255) / 256), 256, 0, c->stream>>>(d_raw, n, c->d_kd, c->n_kernels, c->cfg.n_reasons,
                                                             d_words, d_n_invalid);
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

gs_status hist_run(gs_ctx* c, const uint32_t* d_words, uint64_t n, int32_t* d_hist, unsigned long long* d_n_invalid,
                   int accumulate, bool zero_first) {
  cudaStream_t st = c->stream;
  const uint32_t P = (uint32_t)c->n_instr, nr = c->cfg.n_reasons;
  if (zero_first && !accumulate) GS_CUDA(c, cudaMemsetAsync(d_hist, 0, (uint64_t)P * 32 * 4, st));
  if (!n) return GS_OK;
  if (reinterpret_cast<uintptr_t>(d_words) & 3u) return fail(c, GS_E_INVAL, "sample pointer must be 4-byte aligned");
  int dev_sms = 148;
  cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, c->device);
  // peel the words before the first 16-byte boundary so the main kernels use 128-bit loads
  const uint64_t head = std::min<uint64_t>(n, ((16u - (reinterpret_cast<uintptr_t>(d_words) & 15u)) & 15u) / 4u);
  if (head) {
    k_hist_global<<<1, 32, 0, st>>>(d_words, head, P, nr, d_hist, d_n_invalid);
    count_launch();
    GS_CUDA(c, cudaGetLastError());
    d_words += head;
    n -= head;
    if (!n) return GS_OK;
  }
  const uint64_t compact = (uint64_t)P * nr;
  const uint32_t n_ranges = (uint32_t)std::max<uint64_t>(1, (compact + kTableBins - 1) / kTableBins);
  uint32_t mode = c->cfg.hist_mode;
  if (mode == GS_HIST_AUTO) mode = n_ranges <= kMaxRanges ? GS_HIST_PRIVATE : GS_HIST_WINDOW;
  if (mode == GS_HIST_PRIVATE && n_ranges > 64) mode = GS_HIST_WINDOW;
  c->last_hist_mode = (int)mode;
  if (mode == GS_HIST_GLOBAL) {
    const uint64_t blocks = std::max<uint64_t>(
        1, std::min<uint64_t>((uint64_t)dev_sms * 4, (n + kThreadsGlobal * 4 - 1) / (kThreadsGlobal * 4)));
    k_hist_global<<<(unsigned)blocks, kThreadsGlobal, 0, st>>>(d_words, n, P, nr, d_hist, d_n_invalid);
    count_launch();
    GS_CUDA(c, cudaGetLastError());
    return GS_OK;
  }
  const size_t smem = (size_t)kTableWords * 4;
  const bool dyn = mode == GS_HIST_WINDOW;
  uint64_t chunks;
  if (dyn) {
    chunks = std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)dev_sms, n / (2ull * kTableBins) + 1));
  } else {
    chunks = std::max<uint64_t>(1, (uint64_t)dev_sms / n_ranges);
    chunks = std::min<uint64_t>(chunks, std::max<uint64_t>(1, n / (2ull * kTableBins)));
  }
  uint64_t chunk = (n + chunks - 1) / chunks;
  chunk = (chunk + 3) & ~3ull;
  chunks = (n + chunk - 1) / chunk;
  if (dyn) {
    GS_CUDA(c, cudaFuncSetAttribute(k_hist_smem<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    k_hist_smem<true><<<(unsigned)chunks, kThreadsSmem, smem, st>>>(d_words, n, P, nr, c->d_kd, c->n_kernels, 1, chunk,
                                                                    d_hist, d_n_invalid);
  } else {
    GS_CUDA(c, cudaFuncSetAttribute(k_hist_smem<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    k_hist_smem<false><<<(unsigned)(chunks * n_ranges), kThreadsSmem, smem, st>>>(
        d_words, n, P, nr, c->d_kd, c->n_kernels, n_ranges, chunk, d_hist, d_n_invalid);
  }
  count_launch();
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
