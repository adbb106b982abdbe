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
#include <cstdlib>

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
constexpr uint32_t kTmaTableWords = 41600;  // TMA kernel: 16-bit pairs, 83200 bins (4378 slots at R = 19)

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

// predicated L2 atomic: one instruction, no branch
__device__ __forceinline__ void red_global_add_if(int32_t* addr, uint32_t v, bool p) {
  asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %2, 0;\n\t@q red.relaxed.gpu.global.add.u32 [%0], %1;\n\t}" ::"l"(addr),
               "r"(v), "r"((uint32_t)p)
               : "memory");
}

// 32-bit counters: no return values, no rare path. Per sample: shared atomic on the window slot
// (or the lane's spare word), plus a predicated L2 atomic when the sample is valid but outside the
// window (WINDOW only; PRIVATE leaves it to the CTA that owns that range).
template <bool SPILL_OUT, int N>
__device__ __forceinline__ void count_batch(const uint32_t (&w)[N], uint32_t P, uint32_t nr, uint32_t ws,
                                            uint32_t nslots, uint32_t* tab, uint32_t one, int32_t* H,
                                            uint32_t& bad) {
#pragma unroll
  for (int q = 0; q < N; q++) {
    const uint32_t slot = w[q] >> 5, d = slot - ws, rs = w[q] & 31u;
    const bool rok = rs < nr;
    const bool in = d < nslots && rok;
    atomicAdd(tab + (in ? d * nr + rs : kTableWords + (threadIdx.x & 31u)), one);  // spare: never flushed
    const bool valid = rok && slot < P;
    if (SPILL_OUT) red_global_add_if(H + w[q], one, valid && !in);
    bad += valid ? 0u : 1u;
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

// ---- 16-bit packed variant: two counters per word, twice the bins per window. The increment
// that takes a half from 0x7FFF to 0x8000 (bit 15 flips: (old ^ (old + inc)) & (inc << 15)) drains
// 0x8000 to the global bin, so a half never carries into its neighbour (at most a few thousand
// increments can be in flight per SM between that add and the drain). Counts stay exact.
// rare path of count_batch16, out of line so its address arithmetic is not hoisted into the loop
template <bool SPILL_OUT>
__device__ __noinline__ void slow16(uint32_t w, uint32_t old, uint32_t sh, uint32_t idx, bool in, uint32_t P,
                                    uint32_t nr, uint32_t* tab, int32_t* H, uint32_t* bad) {
  if (!in) {
    if ((w >> 5) < P && (w & 31u) < nr) {
      if (SPILL_OUT) atomicAdd(H + w, 1);
    } else {
      (*bad)++;
    }
    return;
  }
  if (!((old >> sh) & 0x8000u)) return;
  // the half was already >= 0x8000: move 0x8000 of it to the global bin. Several threads may race
  // here; the CAS makes each successful drain subtract exactly 0x8000 once.
  uint32_t v = tab[idx];
  while ((v >> sh) & 0x8000u) {
    const uint32_t prev = atomicCAS(tab + idx, v, v - (0x8000u << sh));
    if (prev == v) {
      atomicAdd(H + w, 0x8000);
      return;
    }
    v = prev;
  }
}

// 16-bit packed counters, two per word. Per sample: one returning shared atomic; the returned old
// value flags a half already at >= 0x8000 (drained in the rare path before it could reach 0xFFFF:
// at most a few thousand increments are in flight per SM), so counts stay exact.
template <bool SPILL_OUT, int N, uint32_t SPARE = kTableWords>
__device__ __forceinline__ void count_batch16(const uint32_t (&w)[N], uint32_t P, uint32_t nr, uint32_t ws,
                                              uint32_t nslots, uint32_t* tab, uint32_t one, int32_t* H,
                                              uint32_t& bad) {
  uint32_t old[N], flag = 0;
#pragma unroll
  for (int q = 0; q < N; q++) {
    const uint32_t d = (w[q] >> 5) - ws, rs = w[q] & 31u;
    const bool in = d < nslots && rs < nr;
    const uint32_t off = d * nr + rs;
    const uint32_t inc = in ? ((off & 1u) ? 0x10000u : one) : 0u;
    const uint32_t idx = in ? (off >> 1) : SPARE + (threadIdx.x & 31u);  // lane's spare word
    old[q] = atomicAdd(tab + idx, inc);
    flag |= (old[q] & (inc << 15)) | (in ? 0u : 1u);
  }
  if (__any_sync(__activemask(), flag)) {  // rare: a half at >= 0x8000, or a sample outside the window
#pragma unroll
    for (int q = 0; q < N; q++) {
      const uint32_t d = (w[q] >> 5) - ws, rs = w[q] & 31u;
      const bool in = d < nslots && rs < nr;
      const uint32_t off = d * nr + rs;
      slow16<SPILL_OUT>(w[q], old[q], (off & 1u) << 4, off >> 1, in, P, nr, tab, H, &bad);
    }
  }
}

// word i holds bins 2i (low half) and 2i + 1 (high half); bin b <-> slot ws + b / nr, reason b % nr
__device__ void flush_table16(uint32_t* tab, uint32_t ws, uint32_t nr, uint32_t nbins, int32_t* H) {
  const uint32_t stride = 2 * blockDim.x, step_q = stride / nr, step_r = stride % nr;
  uint32_t q = (2 * threadIdx.x) / nr, r = (2 * threadIdx.x) % nr;
  for (uint32_t i = threadIdx.x; 2 * i < nbins; i += blockDim.x) {
    const uint32_t v = tab[i];
    if (v) {
      tab[i] = 0;
      if (v & 0xffffu) atomicAdd(H + (uint64_t)(ws + q) * 32u + r, (int32_t)(v & 0xffffu));
      if (v >> 16) {
        const uint32_t q1 = r + 1 == nr ? q + 1 : q, r1 = r + 1 == nr ? 0 : r + 1;
        atomicAdd(H + (uint64_t)(ws + q1) * 32u + r1, (int32_t)(v >> 16));
      }
    }
    q += step_q;
    r += step_r;
    if (r >= nr) { r -= nr; q++; }
  }
}

template <bool P16, bool SPILL_OUT, int N>
__device__ __forceinline__ void count_any(const uint32_t (&w)[N], uint32_t P, uint32_t nr, uint32_t ws,
                                          uint32_t lim, uint32_t* tab, uint32_t one, int32_t* H, uint32_t& bad) {
  if (P16) count_batch16<SPILL_OUT>(w, P, nr, ws, lim, tab, one, H, bad);
  else count_batch<SPILL_OUT>(w, P, nr, ws, lim, tab, one, H, bad);
}

// Tile queue of the WINDOW kernel. Chunk c (CTA c's contiguous share) is cut into tiles of kTile4
// uint4; rng[c] = (head << 32) | stolen counts tiles taken from the front by the owner and from the
// back by other CTAs that finished their own chunk (work stealing keeps all SMs busy to the end
// while each CTA still walks its own chunk front to back, so windows change rarely).
__device__ __forceinline__ uint32_t n_tiles(uint64_t c, uint64_t chunk, uint64_t n) {
  const uint64_t a4 = c * chunk / 4, e = (c + 1) * chunk < n ? (c + 1) * chunk : n, e4 = e / 4;
  return e4 > a4 ? (uint32_t)((e4 - a4 + kTile4 - 1) / kTile4) : 0u;
}

// returns (chunk << 32) | tile, or ~0 when every tile of every chunk has been taken
__device__ unsigned long long grab_tile(unsigned long long* rng, uint32_t me, uint32_t grid, uint64_t chunk,
                                        uint64_t n) {
  const uint32_t mine = n_tiles(me, chunk, n);
  for (;;) {  // own chunk, front to back
    const unsigned long long o = *(volatile unsigned long long*)(rng + me);
    const uint32_t head = (uint32_t)(o >> 32), stolen = (uint32_t)o;
    if (head + stolen >= mine) break;
    if (atomicCAS(rng + me, o, o + (1ull << 32)) == o) return ((unsigned long long)me << 32) | head;
  }
  for (;;) {  // steal from the back of the chunk with the most tiles left
    uint32_t best = grid, best_left = 0;
    for (uint32_t v = 0; v < grid; v++) {
      const unsigned long long o = *(volatile unsigned long long*)(rng + v);
      const uint32_t nt = n_tiles(v, chunk, n), used = (uint32_t)(o >> 32) + (uint32_t)o;
      if (nt > used && nt - used > best_left) { best_left = nt - used; best = v; }
    }
    if (best == grid) return ~0ull;
    const unsigned long long o = *(volatile unsigned long long*)(rng + best);
    const uint32_t nt = n_tiles(best, chunk, n), head = (uint32_t)(o >> 32), stolen = (uint32_t)o;
    if (head + stolen >= nt) continue;
    if (atomicCAS(rng + best, o, o + 1ull) == o) return ((unsigned long long)best << 32) | (nt - 1 - stolen);
  }
}

// DYN = false: PRIVATE (fixed slot range per CTA); DYN = true: WINDOW (window follows the data)
template <bool DYN, bool P16>
__global__ void __launch_bounds__(kThreadsSmem, 1)
    k_hist_smem(const uint32_t* __restrict__ s, uint64_t n, uint32_t P, uint32_t nr, const KDesc* __restrict__ kd,
                uint32_t nk, uint32_t n_ranges, uint64_t chunk, uint32_t one, int32_t* __restrict__ H,
                unsigned long long* d_n_invalid, unsigned long long* rng) {
  extern __shared__ uint32_t tab[];
  __shared__ uint32_t sh_ws[2];
  __shared__ unsigned long long sh_tile[2];
  const uint32_t nslots = (P16 ? 2 * kTableWords : kTableWords) / nr;
  const uint32_t range = DYN ? 0u : blockIdx.x % n_ranges;
  const uint64_t ci = DYN ? blockIdx.x : blockIdx.x / n_ranges;
  uint32_t ws = DYN ? kNoWindow : range * nslots;
  uint32_t lim = DYN ? 0u : min(nslots, P - min(P, ws));  // slots of the window inside [0, P)
  for (uint32_t i = threadIdx.x; i < kTableWords; i += blockDim.x) tab[i] = 0;
  uint32_t bad = 0;
  const uint4* s4 = reinterpret_cast<const uint4*>(s);
  __syncthreads();
  uint64_t t4 = ci * chunk / 4;  // PRIVATE: walk the own chunk
  const uint64_t e_own = (ci + 1) * chunk < n ? (ci + 1) * chunk : n, e4_own = e_own / 4;
  for (uint32_t it = 0;; it++) {
    uint64_t t4e;
    if (DYN) {
      const auto tile_span = [&](unsigned long long tile) {
        const uint64_t c = tile >> 32, ca4 = c * chunk / 4;
        const uint64_t ce = (c + 1) * chunk < n ? (c + 1) * chunk : n;
        t4 = ca4 + (uint64_t)(uint32_t)tile * kTile4;
        t4e = t4 + kTile4 < ce / 4 ? t4 + kTile4 : ce / 4;
      };
      // warp 0 grabs the next tile and picks its window while the CTA counts the current one
      const auto decide = [&](uint32_t buf) {
        unsigned long long tile = 0;
        if (threadIdx.x == 0) tile = grab_tile(rng, blockIdx.x, gridDim.x, chunk, n);
        tile = __shfl_sync(0xffffffffu, tile, 0);
        uint32_t nws = ws;
        if (tile != ~0ull) {
          uint64_t a4, b4;
          {
            const uint64_t c = tile >> 32, ca4 = c * chunk / 4;
            const uint64_t ce = (c + 1) * chunk < n ? (c + 1) * chunk : n;
            a4 = ca4 + (uint64_t)(uint32_t)tile * kTile4;
            b4 = a4 + kTile4 < ce / 4 ? a4 + kTile4 : ce / 4;
          }
          // window: around the median slot of 32 evenly spaced samples (robust to the cold tail
          // of a kernel's samples); the whole kernel if it fits
          const uint32_t w = __ldg(s + 4 * (a4 + (b4 - a4) * threadIdx.x / 32));
          const bool ok = (w >> 5) < P && (w & 31u) < nr;
          const uint32_t slot = ok ? (w >> 5) : 0xffffffffu;
          uint32_t le = 0;  // lanes whose slot is <= mine
          for (int j = 0; j < 32; j++) le += __shfl_sync(0xffffffffu, slot, j) <= slot ? 1u : 0u;
          const uint32_t nvalid = __popc(__ballot_sync(0xffffffffu, ok));
          // median: the smallest valid slot with more than half of the valid samples at or below it
          const uint32_t med = __reduce_min_sync(0xffffffffu, ok && 2 * le > nvalid ? slot : 0xffffffffu);
          if (med != 0xffffffffu && (ws == kNoWindow || med - ws >= nslots || med - ws < nslots / 8 ||
                                     med - ws >= nslots - nslots / 8)) {
            uint32_t lo = 0, hi = nk;  // kernel of the slot: last k with first <= slot
            while (hi - lo > 1) {
              const uint32_t mid = (lo + hi) >> 1;
              if (__ldg(&kd[mid].first) <= med) lo = mid;
              else hi = mid;
            }
            const KDesc K = kd[lo];
            uint32_t cws;
            if (K.n <= nslots) cws = K.first;                       // the whole kernel fits
            else {                                                  // centre on the median, inside the kernel
              cws = med > nslots / 2 ? med - nslots / 2 : 0;
              cws = min(max(cws, K.first), K.first + K.n - nslots);
            }
            if (ws == kNoWindow || cws != ws) nws = cws;
          }
        }
        if (nws == kNoWindow) nws = 0;
        if (threadIdx.x == 0) {
          sh_tile[buf] = tile;
          sh_ws[buf] = nws;
        }
      };
      if (it == 0 && threadIdx.x < 32) decide(0);
      __syncthreads();
      const unsigned long long tile = sh_tile[it & 1];
      if (tile == ~0ull) break;
      tile_span(tile);
      const uint32_t nws = sh_ws[it & 1];
      if (nws != ws) {
        if (ws != kNoWindow) {
          if (P16) flush_table16(tab, ws, nr, lim * nr, H);
          else flush_table(tab, ws, nr, lim * nr, H);
          __syncthreads();
        }
        ws = nws;
        lim = min(nslots, P - min(P, ws));
      }
      if (threadIdx.x < 32) decide((it + 1) & 1);
    } else {
      if (t4 >= e4_own) break;
      t4e = t4 + kTile4 < e4_own ? t4 + kTile4 : e4_own;
    }
    uint64_t i = t4 + threadIdx.x;
    for (; i + (kVec - 1) * blockDim.x < t4e; i += kVec * blockDim.x) {  // kVec 128-bit loads in flight
      uint32_t w[4 * kVec];
#pragma unroll
      for (int u = 0; u < kVec; u++) {
        const uint4 v = __ldg(s4 + i + u * blockDim.x);
        w[4 * u] = v.x; w[4 * u + 1] = v.y; w[4 * u + 2] = v.z; w[4 * u + 3] = v.w;
      }
      if (P16) {  // returning atomics: batches of 4 keep the old values in registers
#pragma unroll
        for (int u = 0; u < kVec; u++) {
          const uint32_t wq[4] = {w[4 * u], w[4 * u + 1], w[4 * u + 2], w[4 * u + 3]};
          count_any<P16, DYN>(wq, P, nr, ws, lim, tab, one, H, bad);
        }
      } else {
        count_any<P16, DYN>(w, P, nr, ws, lim, tab, one, H, bad);
      }
    }
    for (; i < t4e; i += blockDim.x) {
      const uint4 v = __ldg(s4 + i);
      const uint32_t w[4] = {v.x, v.y, v.z, v.w};
      count_any<P16, DYN>(w, P, nr, ws, lim, tab, one, H, bad);
    }
    if (!DYN) t4 = t4e;
  }
  // the last chunk's words after its last 16-byte boundary (< 4 words), counted by its owner
  if (e_own == n) {
    if (DYN && ws == kNoWindow) {  // a window is needed even if no tile was processed
      ws = 0;
      lim = min(nslots, P);
    }
    for (uint64_t i = e4_own * 4 + threadIdx.x; i < n; i += blockDim.x) {
      const uint32_t w[1] = {s[i]};
      count_any<P16, DYN>(w, P, nr, ws, lim, tab, one, H, bad);
    }
  }
  if (range == 0) count_invalid(bad, d_n_invalid);
  __syncthreads();
  if (ws != kNoWindow) {
    if (P16) flush_table16(tab, ws, nr, lim * nr, H);
    else flush_table(tab, ws, nr, lim * nr, H);
  }
}

// =============================================================================== TMA-fed WINDOW kernel
// Warp-specialised: warp 0 is the producer (tile queue, window choice, TMA bulk copies of sample
// stages into shared memory); warps 1..31 consume one 128-bit word (4 samples) each per stage.
// kStages stages of kStage4 uint4 keep ~62 KB of samples in flight per SM independently of
// registers (the register-fed kernel was memory-latency bound: 57% long-scoreboard stalls).
constexpr int kConsumerWarps = 31;
constexpr uint32_t kStage4 = kConsumerWarps * 32;          // uint4 per stage: one per consumer thread
constexpr uint32_t kStageBytes = kStage4 * 16;             // 15872 B
constexpr int kStages = 4;
constexpr size_t kTmaSmem = (size_t)kStages * kStageBytes + (size_t)(kTmaTableWords + 32) * 4;

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(unsigned long long* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(unsigned long long* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_tx(unsigned long long* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(unsigned long long* b, uint32_t parity) {
  uint32_t done = 0;
  while (!done)
    asm volatile("{\n\t.reg .pred p;\n\tmbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n\tselp.u32 %0, 1, 0, p;\n\t}"
                 : "=r"(done)
                 : "r"(smem_u32(b)), "r"(parity)
                 : "memory");
}
__device__ __forceinline__ void tma_load(void* dst, const void* src, uint32_t bytes, unsigned long long* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void consumer_sync() { asm volatile("bar.sync 1, %0;" ::"r"(kConsumerWarps * 32) : "memory"); }

// flush helpers over an explicit thread range [0, nt)
__device__ void flush_pairs(uint32_t* tab, uint32_t words, uint32_t ws, uint32_t nr, uint32_t nbins, int32_t* H,
                            uint32_t t, uint32_t nt) {
  const uint32_t stride = 2 * nt, step_q = stride / nr, step_r = stride % nr;
  uint32_t q = (2 * t) / nr, r = (2 * t) % nr;
  for (uint32_t i = t; i < words && 2 * i < nbins; i += nt) {
    const uint32_t v = tab[i];
    if (v) {
      tab[i] = 0;
      if (v & 0xffffu) atomicAdd(H + (uint64_t)(ws + q) * 32u + r, (int32_t)(v & 0xffffu));
      if (v >> 16) {
        const uint32_t q1 = r + 1 == nr ? q + 1 : q, r1 = r + 1 == nr ? 0 : r + 1;
        atomicAdd(H + (uint64_t)(ws + q1) * 32u + r1, (int32_t)(v >> 16));
      }
    }
    q += step_q;
    r += step_r;
    if (r >= nr) { r -= nr; q++; }
  }
}

__global__ void __launch_bounds__(32 * (kConsumerWarps + 1), 1)
    k_hist_tma(const uint32_t* __restrict__ s, uint64_t n, uint32_t P, uint32_t nr, const KDesc* __restrict__ kd,
               uint32_t nk, uint64_t chunk, uint32_t one, int32_t* __restrict__ H, unsigned long long* d_n_invalid,
               unsigned long long* rng) {
  extern __shared__ __align__(128) uint8_t dyn[];
  uint4* stage = reinterpret_cast<uint4*>(dyn);
  uint32_t* tab = reinterpret_cast<uint32_t*>(dyn + (size_t)kStages * kStageBytes);
  __shared__ __align__(8) unsigned long long full_bar[kStages], empty_bar[kStages];
  __shared__ uint32_t meta_ws[kStages], meta_cnt[kStages];
  const uint32_t nslots = 2 * kTmaTableWords / nr;
  const uint32_t warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  for (uint32_t i = threadIdx.x; i < kTmaTableWords + 32; i += blockDim.x) tab[i] = 0;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kStages; i++) {
      mbar_init(full_bar + i, 1);
      mbar_init(empty_bar + i, kConsumerWarps);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
  }
  __syncthreads();
  const uint4* s4 = reinterpret_cast<const uint4*>(s);
  const uint64_t e_own = (blockIdx.x + 1) * chunk < n ? (blockIdx.x + 1) * chunk : n;
  if (warp == 0) {
    // ------------------------------------------------------------------ producer
    uint32_t ws = kNoWindow, st = 0;
    for (;;) {
      unsigned long long tile = 0;
      if (lane == 0) tile = grab_tile(rng, blockIdx.x, gridDim.x, chunk, n);
      tile = __shfl_sync(0xffffffffu, tile, 0);
      if (tile == ~0ull) break;
      const uint64_t c = tile >> 32, ca4 = c * chunk / 4;
      const uint64_t ce = (c + 1) * chunk < n ? (c + 1) * chunk : n;
      const uint64_t t4 = ca4 + (uint64_t)(uint32_t)tile * kTile4;
      const uint64_t t4e = t4 + kTile4 < ce / 4 ? t4 + kTile4 : ce / 4;
      if (t4e <= t4) continue;
      {  // window: around the median slot of 32 evenly spaced samples; the whole kernel if it fits
        const uint32_t w = __ldg(s + 4 * (t4 + (t4e - t4) * lane / 32));
        const bool ok = (w >> 5) < P && (w & 31u) < nr;
        const uint32_t slot = ok ? (w >> 5) : 0xffffffffu;
        uint32_t le = 0;
        for (int j = 0; j < 32; j++) le += __shfl_sync(0xffffffffu, slot, j) <= slot ? 1u : 0u;
        const uint32_t nvalid = __popc(__ballot_sync(0xffffffffu, ok));
        const uint32_t med = __reduce_min_sync(0xffffffffu, ok && 2 * le > nvalid ? slot : 0xffffffffu);
        if (med != 0xffffffffu && (ws == kNoWindow || med - ws >= nslots || med - ws < nslots / 8 ||
                                   med - ws >= nslots - nslots / 8)) {
          uint32_t lo = 0, hi = nk;
          while (hi - lo > 1) {
            const uint32_t mid = (lo + hi) >> 1;
            if (__ldg(&kd[mid].first) <= med) lo = mid;
            else hi = mid;
          }
          const KDesc K = kd[lo];
          uint32_t cws;
          if (K.n <= nslots) cws = K.first;
          else {
            cws = med > nslots / 2 ? med - nslots / 2 : 0;
            cws = min(max(cws, K.first), K.first + K.n - nslots);
          }
          ws = cws;
        }
        if (ws == kNoWindow) ws = 0;
      }
      for (uint64_t p = t4; p < t4e; p += kStage4, st++) {
        const uint32_t cnt = t4e - p < kStage4 ? (uint32_t)(t4e - p) : kStage4;
        const uint32_t sb = st % kStages;
        if (st >= (uint32_t)kStages) mbar_wait(empty_bar + sb, ((st / kStages) + 1) & 1);
        if (lane == 0) {
          meta_ws[sb] = ws;
          meta_cnt[sb] = cnt;
          mbar_arrive_tx(full_bar + sb, cnt * 16);
          tma_load(stage + (size_t)sb * kStage4, s4 + p, cnt * 16, full_bar + sb);
        }
        __syncwarp();
      }
    }
    const uint32_t sb = st % kStages;  // end marker
    if (st >= (uint32_t)kStages) mbar_wait(empty_bar + sb, ((st / kStages) + 1) & 1);
    if (lane == 0) {
      meta_cnt[sb] = 0;
      mbar_arrive(full_bar + sb);
    }
    return;
  }
  // -------------------------------------------------------------------- consumers
  const uint32_t ct = threadIdx.x - 32, nct = kConsumerWarps * 32;
  uint32_t ws = kNoWindow, lim = 0, bad = 0;
  for (uint32_t st = 0;; st++) {
    const uint32_t sb = st % kStages;
    mbar_wait(full_bar + sb, (st / kStages) & 1);
    const uint32_t cnt = meta_cnt[sb], nws = meta_ws[sb];
    if (cnt == 0) break;
    if (nws != ws) {  // window change: every consumer has finished the previous stages
      consumer_sync();
      if (ws != kNoWindow) flush_pairs(tab, kTmaTableWords, ws, nr, lim * nr, H, ct, nct);
      consumer_sync();
      ws = nws;
      lim = min(nslots, P - min(P, ws));
    }
    const uint4 v = ct < cnt ? stage[(size_t)sb * kStage4 + ct] : make_uint4(0, 0, 0, 0);
    __syncwarp();
    if (lane == 0) mbar_arrive(empty_bar + sb);  // stage may be refilled; the data is in registers
    if (ct < cnt) {
      const uint32_t w[4] = {v.x, v.y, v.z, v.w};
      count_batch16<true, 4, kTmaTableWords>(w, P, nr, ws, lim, tab, one, H, bad);
    }
  }
  // the last chunk's words after its last 16-byte boundary (< 4): L2 atomics
  if (e_own == n)
    for (uint64_t i = (n / 4) * 4 + ct; i < n; i += nct) {
      const uint32_t w = s[i];
      if ((w >> 5) < P && (w & 31u) < nr) atomicAdd(H + w, 1);
      else bad++;
    }
  for (int o = 16; o; o >>= 1) bad += __shfl_xor_sync(0xffffffffu, bad, o);
  if (lane == 0 && bad) atomicAdd(d_n_invalid, (unsigned long long)bad);
  consumer_sync();
  if (ws != kNoWindow) flush_pairs(tab, kTmaTableWords, ws, nr, lim * nr, H, ct, nct);
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
  const uint32_t nslots32 = kTableWords / nr, nslots16 = 2 * kTableWords / nr;  // whole slots per window
  const auto ranges = [&](uint32_t ns) { return (uint32_t)std::max<uint64_t>(1, ((uint64_t)P + ns - 1) / ns); };
  uint32_t max_kn = 0;
  for (const auto& K : c->kd_h) max_kn = std::max(max_kn, K.n);
  uint32_t mode = c->cfg.hist_mode, bits = c->cfg.hist_counter_bits;
  if (mode == GS_HIST_AUTO) {
    if (ranges(bits == 16 ? nslots16 : nslots32) <= kMaxRanges) mode = GS_HIST_PRIVATE;
    else if (!bits && ranges(nslots16) <= kMaxRanges) { mode = GS_HIST_PRIVATE; bits = 16; }
    else mode = GS_HIST_WINDOW;
  }
  if (!bits) bits = (mode == GS_HIST_WINDOW && max_kn > nslots32) ? 16 : 32;  // whole kernels per window
  const uint32_t n_ranges = ranges(bits == 16 ? nslots16 : nslots32);
  if (mode == GS_HIST_PRIVATE && n_ranges > 64) mode = GS_HIST_WINDOW;
  c->last_hist_bits = (int)bits;
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
  if (dyn) {  // work-stealing tile queue, one 64-bit word per chunk
    GS_CUDA(c, dev_grow(&c->d_tileq, &c->tileq_cap, chunks));
    GS_CUDA(c, cudaMemsetAsync(c->d_tileq, 0, chunks * 8, st));
  }
  auto launch = [&](auto kern, uint32_t grid, uint32_t nrg) -> gs_status {
    GS_CUDA(c, cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    kern<<<grid, kThreadsSmem, smem, st>>>(d_words, n, P, nr, c->d_kd, c->n_kernels, nrg, chunk, 1u, d_hist,
                                           d_n_invalid, c->d_tileq);
    return GS_OK;
  };
  gs_status ls;
  if (dyn && bits == 16 && getenv("GS_HIST_TMA")) {  // TMA-fed warp-specialised kernel (opt-in)
    GS_CUDA(c, cudaFuncSetAttribute(k_hist_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kTmaSmem));
    k_hist_tma<<<(uint32_t)chunks, 32 * (kConsumerWarps + 1), kTmaSmem, st>>>(
        d_words, n, P, nr, c->d_kd, c->n_kernels, chunk, 1u, d_hist, d_n_invalid, c->d_tileq);
    ls = GS_OK;
  } else if (dyn) ls = bits == 16 ? launch(k_hist_smem<true, true>, (uint32_t)chunks, 1u)
                           : launch(k_hist_smem<true, false>, (uint32_t)chunks, 1u);
  else ls = bits == 16 ? launch(k_hist_smem<false, true>, (uint32_t)(chunks * n_ranges), n_ranges)
                       : launch(k_hist_smem<false, false>, (uint32_t)(chunks * n_ranges), n_ranges);
  if (ls != GS_OK) return ls;
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

void attrib_free(gs_ctx* c) {
  if (c->d_tileq) cudaFree(c->d_tileq);
  c->d_tileq = nullptr;
  c->tileq_cap = 0;
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
