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
constexpr uint32_t kTableWords = 56 * 1024 - 32;   // 224 KB of shared memory: 32-bit counters + 32 spares
constexpr uint32_t kMaxRanges = 3;
constexpr uint32_t kTile4 = 65536;                 // uint4 per window decision (256K samples)
constexpr int kVec = 4;                            // 128-bit loads in flight per thread
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
// The table holds kTableWords 32-bit counters for the compact bins of a window of whole slots
// [ws, ws + nslots), nslots = kTableWords / n_reasons: counter index (slot - ws) * n_reasons + reason.
// Fast path per sample (8 instructions): d = (w >> 5) - ws; in = d < nslots && (w & 31) < nr;
// smem[d * nr + (w & 31)] += 1 (no return value). Lanes outside the window take a warp-uniform
// slow path: L2 atomic (WINDOW) / skip (PRIVATE: another CTA owns that range) / invalid count.

template <bool SPILL_OUT>
__device__ __forceinline__ void slow_one(uint32_t w, uint32_t P, uint32_t nr, int32_t* H, uint32_t& bad) {
  if ((w >> 5) < P && (w & 31u) < nr) {
    if (SPILL_OUT) atomicAdd(H + w, 1);
  } else {
    bad++;
  }
}

// predicated shared-memory add of `one` (a run-time 1, so ptxas emits one predicated ATOMS.ADD
// instead of a branch around ATOMS.POPC.INC)
__device__ __forceinline__ void red_shared_add_if(uint32_t addr, uint32_t one, bool p) {
  asm volatile(
      "{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q red.shared.add.u32 [%0], %1;\n\t}" ::"r"(addr), "r"(one),
      "r"((uint32_t)p)
      : "memory");
}

template <bool SPILL_OUT, int N>
__device__ __forceinline__ void count_batch(const uint32_t (&w)[N], uint32_t P, uint32_t nr, uint32_t ws,
                                            uint32_t nslots, uint32_t* tab, uint32_t one, int32_t* H,
                                            uint32_t& bad) {
  uint32_t n_out = 0;
#pragma unroll
  for (int q = 0; q < N; q++) {
    const uint32_t d = (w[q] >> 5) - ws, rs = w[q] & 31u;
    const bool in = d < nslots && rs < nr;
    // unconditional shared atomic: lanes outside the window add 0 to a spare word (no branch)
    atomicAdd(tab + (in ? d * nr + rs : kTableWords + (threadIdx.x & 31u)), in ? one : 0u);
    n_out += in ? 0u : 1u;
  }
  if (__any_sync(__activemask(), n_out)) {  // rare: some lane saw a sample outside the window
#pragma unroll
    for (int q = 0; q < N; q++) {
      const uint32_t d = (w[q] >> 5) - ws, rs = w[q] & 31u;
      if (!(d < nslots && rs < nr)) slow_one<SPILL_OUT>(w[q], P, nr, H, bad);
    }
  }
}

// flush the window's counters into H and zero them; word i <-> slot ws + i / nr, reason i % nr
__device__ void flush_table(uint32_t* tab, uint32_t ws, uint32_t nr, uint32_t nwords, int32_t* H) {
  const uint32_t step_q = blockDim.x / nr, step_r = blockDim.x % nr;
  uint32_t q = threadIdx.x / nr, r = threadIdx.x % nr;
  for (uint32_t i = threadIdx.x; i < nwords; i += blockDim.x) {
    const uint32_t v = tab[i];
    if (v) {
      tab[i] = 0;
      atomicAdd(H + (uint64_t)(ws + q) * 32u + r, (int32_t)v);
    }
    q += step_q;
    r += step_r;
    if (r >= nr) { r -= nr; q++; }
  }
}

// DYN = false: PRIVATE (fixed slot range per CTA); DYN = true: WINDOW (window follows the data)
template <bool DYN>
__global__ void __launch_bounds__(kThreadsSmem, 1)
    k_hist_smem(const uint32_t* __restrict__ s, uint64_t n, uint32_t P, uint32_t nr, const KDesc* __restrict__ kd,
                uint32_t nk, uint32_t n_ranges, uint64_t chunk, uint32_t one, int32_t* __restrict__ H,
                unsigned long long* d_n_invalid) {
  extern __shared__ uint32_t tab[];
  __shared__ uint32_t sh_ws[2];
  const uint32_t nslots = kTableWords / nr, nwords = nslots * nr;
  const uint32_t tab_s = (uint32_t)__cvta_generic_to_shared(tab);
  const uint32_t range = DYN ? 0u : blockIdx.x % n_ranges;
  const uint64_t ci = DYN ? blockIdx.x : blockIdx.x / n_ranges;
  uint32_t ws = DYN ? kNoWindow : range * nslots;
  uint32_t lim = DYN ? 0u : min(nslots, P - min(P, ws));  // slots of the window inside [0, P)
  for (uint32_t i = threadIdx.x; i < nwords; i += blockDim.x) tab[i] = 0;
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
      if (threadIdx.x < 32) {
        // window for this tile: around the median slot of 32 evenly spaced samples (robust to the
        // cold tail of a kernel's samples); whole kernel if it fits
        const uint64_t span = t4e - t4;
        const uint32_t w = s[4 * (t4 + span * threadIdx.x / 32)];
        const bool ok = (w >> 5) < P && (w & 31u) < nr;
        const uint32_t slot = ok ? (w >> 5) : 0xffffffffu;
        uint32_t le = 0;  // lanes whose slot is <= mine
        for (int j = 0; j < 32; j++) le += __shfl_sync(0xffffffffu, slot, j) <= slot ? 1u : 0u;
        const uint32_t nvalid = __popc(__ballot_sync(0xffffffffu, ok));
        // median: the smallest valid slot with more than half of the valid samples at or below it
        const uint32_t med = __reduce_min_sync(0xffffffffu, ok && 2 * le > nvalid ? slot : 0xffffffffu);
        if (threadIdx.x == 0) {
          uint32_t nws = ws;
          if (med != 0xffffffffu && (ws == kNoWindow || med - ws >= nslots || med - ws < nslots / 8 ||
                                     med - ws >= nslots - nslots / 8)) {
            uint32_t lo = 0, hi = nk;  // kernel of the slot: last k with first <= slot
            while (hi - lo > 1) {
              const uint32_t mid = (lo + hi) >> 1;
              if (kd[mid].first <= med) lo = mid;
              else hi = mid;
            }
            const KDesc K = kd[lo];
            uint32_t c;
            if (K.n <= nslots) c = K.first;                         // the whole kernel fits
            else {                                                  // centre on the median, inside the kernel
              c = med > nslots / 2 ? med - nslots / 2 : 0;
              c = min(max(c, K.first), K.first + K.n - nslots);
            }
            // keep the current window when the new one would not move it (already centred)
            if (ws == kNoWindow || c != ws) nws = c;
          }
          if (nws == kNoWindow) nws = 0;
          sh_ws[it & 1] = nws;
        }
      }
      __syncthreads();
      const uint32_t nws = sh_ws[it & 1];
      if (nws != ws) {
        if (ws != kNoWindow) {
          flush_table(tab, ws, nr, lim * nr, H);
          __syncthreads();
        }
        ws = nws;
        lim = min(nslots, P - min(P, ws));
      }
    }
    uint64_t i = t4 + threadIdx.x;
    for (; i + (kVec - 1) * blockDim.x < t4e; i += kVec * blockDim.x) {  // kVec 128-bit loads in flight
      uint32_t w[4 * kVec];
#pragma unroll
      for (int u = 0; u < kVec; u++) {
        const uint4 v = __ldg(s4 + i + u * blockDim.x);
        w[4 * u] = v.x; w[4 * u + 1] = v.y; w[4 * u + 2] = v.z; w[4 * u + 3] = v.w;
      }
      count_batch<DYN>(w, P, nr, ws, lim, tab, one, H, bad);
    }
    for (; i < t4e; i += blockDim.x) {
      const uint4 v = __ldg(s4 + i);
      const uint32_t w[4] = {v.x, v.y, v.z, v.w};
      count_batch<DYN>(w, P, nr, ws, lim, tab, one, H, bad);
    }
  }
  for (uint64_t i = e4 * 4 + threadIdx.x; i < e; i += blockDim.x) {
    const uint32_t w[1] = {s[i]};
    count_batch<DYN>(w, P, nr, ws, lim, tab, one, H, bad);
  }
  if (range == 0) count_invalid(bad, d_n_invalid);
  __syncthreads();
  if (ws != kNoWindow) flush_table(tab, ws, nr, min(nwords, lim * nr), H);
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
  const uint32_t nslots = kTableWords / nr;  // whole slots per shared-memory window
  const uint32_t n_ranges = (uint32_t)std::max<uint64_t>(1, ((uint64_t)P + nslots - 1) / nslots);
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
  const size_t smem = (size_t)(kTableWords + 32) * 4;  // + one spare word per lane
  const bool dyn = mode == GS_HIST_WINDOW;
  uint64_t chunks;
  if (dyn) {
    chunks = std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)dev_sms, n / (2ull * kTableWords) + 1));
  } else {
    chunks = std::max<uint64_t>(1, (uint64_t)dev_sms / n_ranges);
    chunks = std::min<uint64_t>(chunks, std::max<uint64_t>(1, n / (2ull * kTableWords)));
  }
  uint64_t chunk = (n + chunks - 1) / chunks;
  chunk = (chunk + 3) & ~3ull;
  chunks = (n + chunk - 1) / chunk;
  if (dyn) {
    GS_CUDA(c, cudaFuncSetAttribute(k_hist_smem<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    k_hist_smem<true><<<(unsigned)chunks, kThreadsSmem, smem, st>>>(d_words, n, P, nr, c->d_kd, c->n_kernels, 1, chunk,
                                                                    1u, d_hist, d_n_invalid);
  } else {
    GS_CUDA(c, cudaFuncSetAttribute(k_hist_smem<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    k_hist_smem<false><<<(unsigned)(chunks * n_ranges), kThreadsSmem, smem, st>>>(
        d_words, n, P, nr, c->d_kd, c->n_kernels, n_ranges, chunk, 1u, d_hist, d_n_invalid);
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
