// attrib.cu — PC-sample packing and the per-PC x stall-reason histogram
// (§2.2, §3).
//
// Packed sample word = compact bin  cb = slot * R + reason  (slot = first_slot[kernel] + pc/16,
// R = n_reasons active reasons; R30). Valid iff cb < P * R. The histogram H is int32 [P][row]
// (row = gs_config.hist_row: 32, or R for compact rows); bin (slot, reason) lives at
// H[slot * row + reason] — with compact rows that is H[cb].
//
// Global atomics alone run at 50-200 G samples/s on B200 (profiles/r01_atomics_microbench.txt),
// far below the ~1.6 T samples/s HBM streams 4-byte samples at, so counting happens in shared
// memory over a WINDOW of whole slots [ws, ws + nslots): table word (cb - ws*R) (32-bit counters)
// or half (cb - ws*R) (16-bit counters, two per word). The compact word makes the per-sample fast
// path tiny: off = cb - wb; in = off < lim; shared atomic on tab[in ? off : spare(lane)].
// Samples outside the window (rare) take an out-of-line path after one warp vote per batch.
//
// 16-bit counters are exact: the returned old value flags a half that is already >= 0x8000; the
// rare path moves 0x8000 of it to the global bin with a CAS, long before it could reach 0xFFFF
// (at most a few thousand increments are in flight per SM).
//
// Strategies (gs_config.hist_mode):
//   PRIVATE  fixed slot ranges per CTA (the CTAs of one sample chunk are adjacent in launch
//            order, so the re-reads of a chunk hit L2); used when the bins fit in <= 3 windows.
//   WINDOW   one persistent CTA per SM; tiles of the sample stream come from a per-CTA queue
//            with work stealing; the window follows the data (median slot of 32 samples of the
//            next tile, decided by warp 0 while the CTA counts the current tile; the sample's
//            whole kernel when it fits). Suited to PC-sampling traces, which arrive grouped by
//            kernel launch.
//   GLOBAL   one L2 atomic per valid sample (reference strategy).
#include <cuda_runtime.h>

#include <algorithm>

#include "ctx.h"

namespace gs {
namespace {

constexpr int kThreadsGlobal = 512;
#ifndef GS_HIST_THREADS
#define GS_HIST_THREADS 1024
#endif
#ifndef GS_KVEC
#define GS_KVEC 8
#endif
constexpr int kThreads = GS_HIST_THREADS;
#ifndef GS_TABLE_WORDS
#define GS_TABLE_WORDS (56 * 1024 - 32)
#endif
constexpr uint32_t kTableWords = GS_TABLE_WORDS;   // + 32 spare words (one per lane) = 224 KB
constexpr uint32_t kMaxRanges = 3;
constexpr uint32_t kMinTableWords = 8192;          // smallest WINDOW table (32 KB)
#ifndef GS_TILE4
#define GS_TILE4 (4 * GS_KVEC * (GS_HIST_THREADS - 32))
#endif
constexpr uint32_t kTile4 = GS_TILE4;              // uint4 per WINDOW tile: 4 batches of the counters

constexpr int kVec = GS_KVEC;                          // 128-bit loads in flight per thread
constexpr uint32_t kNoWindow = 0xffffffffu;

// x / d for x < 2^32, 1 <= d <= 32: floor(x * ceil(2^40 / d) / 2^40) (error < 2^37 / 2^40 < 1/d);
// row = bins per H row (32, or d for compact rows)
struct Div {
  uint64_t m;
  uint32_t d;
  uint32_t row;
};
__host__ __device__ inline Div make_div(uint32_t d, uint32_t row) { return Div{((1ull << 40) + d - 1) / d, d, row}; }
__device__ __forceinline__ uint32_t divq(uint32_t x, Div v) { return (uint32_t)(((unsigned __int128)x * v.m) >> 40); }
// H index of a compact bin (the bin itself when rows are compact)
__device__ __forceinline__ uint64_t hidx(uint32_t cb, Div v) {
  if (v.row == v.d) return cb;
  const uint32_t q = divq(cb, v);
  return (uint64_t)q * v.row + (cb - q * v.d);
}

__device__ __forceinline__ void count_invalid(uint32_t n_bad, unsigned long long* d_n_invalid) {
  for (int o = 16; o; o >>= 1) n_bad += __shfl_xor_sync(0xffffffffu, n_bad, o);
  if ((threadIdx.x & 31) == 0 && n_bad) atomicAdd(d_n_invalid, (unsigned long long)n_bad);
}

// one raw record (kernel, pc offset, reason) -> packed word (~0u if invalid, R30)
__device__ __forceinline__ uint32_t pack1(uint32_t k, uint32_t pc, uint32_t reason, const KDesc* __restrict__ kd,
                                          uint32_t nk, uint32_t nr, uint32_t& bad) {
  bool ok = k < nk && (pc & 15u) == 0 && reason < nr;
  uint32_t w = 0xffffffffu;
  if (ok) {
    const KDesc K = kd[k];
    ok = (pc >> 4) < K.n;
    if (ok) w = (K.first + (pc >> 4)) * nr + reason;
  }
  bad += ok ? 0u : 1u;
  return w;
}

// N1: four records (48 B = three 128-bit loads) -> one 128-bit store per thread, grid-stride over
// the 16-byte-aligned body; the < 4 trailing records and an unaligned input take the scalar loop
__global__ void __launch_bounds__(256) k_pack(const uint32_t* __restrict__ raw, uint64_t n, const KDesc* __restrict__ kd,
                                              uint32_t nk, uint32_t nr, uint32_t* __restrict__ words,
                                              unsigned long long* d_n_invalid) {
  uint32_t bad = 0;
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t t0 = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  const bool vec = ((reinterpret_cast<uintptr_t>(raw) | reinterpret_cast<uintptr_t>(words)) & 15u) == 0;
  const uint64_t n4 = vec ? n / 4 : 0;
  const uint4* r4 = reinterpret_cast<const uint4*>(raw);
  uint4* w4 = reinterpret_cast<uint4*>(words);
  for (uint64_t i = t0; i < n4; i += stride) {
    const uint4 a = __ldcs(r4 + 3 * i), b = __ldcs(r4 + 3 * i + 1), c = __ldcs(r4 + 3 * i + 2);
    uint4 o;
    o.x = pack1(a.x, a.y, a.z, kd, nk, nr, bad);
    o.y = pack1(a.w, b.x, b.y, kd, nk, nr, bad);
    o.z = pack1(b.z, b.w, c.x, kd, nk, nr, bad);
    o.w = pack1(c.y, c.z, c.w, kd, nk, nr, bad);
    __stcs(w4 + i, o);
  }
  for (uint64_t i = 4 * n4 + t0; i < n; i += stride) words[i] = pack1(raw[3 * i], raw[3 * i + 1], raw[3 * i + 2], kd, nk, nr, bad);
  count_invalid(bad, d_n_invalid);
}

// Pre-aggregated records {kernel, pc, reason, count} (CUPTI PC-sampling shape): one 128-bit load
// per record, one L2 atomic per valid record (records are already one per (pc, reason), so there
// is nothing to privatise); invalid records add their count to n_invalid.
__global__ void k_counts(const uint4* __restrict__ rec, uint64_t n, const KDesc* __restrict__ kd, uint32_t nk,
                         uint32_t nr, uint32_t row, int32_t* __restrict__ H, unsigned long long* d_n_invalid) {
  unsigned long long bad = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint4 r = __ldg(rec + i);  // x kernel, y pc, z reason, w count
    bool ok = r.x < nk && (r.y & 15u) == 0 && r.z < nr;
    uint32_t first = 0;
    if (ok) {
      const KDesc K = kd[r.x];
      ok = (r.y >> 4) < K.n;
      first = K.first;
    }
    if (ok) {
      if (r.w) atomicAdd(H + (uint64_t)(first + (r.y >> 4)) * row + r.z, (int32_t)r.w);
    } else {
      bad += r.w;
    }
  }
  for (int o = 16; o; o >>= 1) bad += __shfl_xor_sync(0xffffffffu, bad, o);
  if ((threadIdx.x & 31) == 0 && bad) atomicAdd(d_n_invalid, bad);
}

// Pre-aggregated records already packed on the host as {compact bin, count} (8 B; the CUPTI
// ingest validates and packs while it flattens): one L2 atomic per record with a count; a bin >=
// P * R is invalid and adds its count to n_invalid.
__global__ void k_counts8(const uint2* __restrict__ rec, uint64_t n, uint32_t pnr, Div dv, int32_t* __restrict__ H,
                          unsigned long long* d_n_invalid) {
  unsigned long long bad = 0;
  for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint2 r = __ldg(rec + i);  // x bin, y count
    if (r.x < pnr) {
      if (r.y) atomicAdd(H + hidx(r.x, dv), (int32_t)r.y);
    } else {
      bad += r.y;
    }
  }
  for (int o = 16; o; o >>= 1) bad += __shfl_xor_sync(0xffffffffu, bad, o);
  if ((threadIdx.x & 31) == 0 && bad) atomicAdd(d_n_invalid, bad);
}

// -------------------------------------------------------------------------------- GLOBAL
__global__ void __launch_bounds__(kThreadsGlobal) k_hist_global(const uint32_t* __restrict__ s, uint64_t n,
                                                                uint32_t pnr, Div dv, int32_t* __restrict__ H,
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
      if (w[q] < pnr) atomicAdd(H + hidx(w[q], dv), 1);
      else bad++;
    }
  }
  for (uint64_t i = n4 * 4 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += stride) {
    if (s[i] < pnr) atomicAdd(H + hidx(s[i], dv), 1);
    else bad++;
  }
  count_invalid(bad, d_n_invalid);
}

// -------------------------------------------------------------------------------- shared-memory table
struct Win {
  uint32_t wb;   // first compact bin of the window (ws * R)
  uint32_t lim;  // bins of the window inside [0, P * R)
};

// Where a sample outside the window goes: OUT_DROP (PRIVATE: another CTA owns that range), OUT_RED
// (L2 atomic), OUT_DEFER (WINDOW: appended to the CTA's ring, counted after the next window switch).
enum { OUT_DROP = 0, OUT_RED = 1, OUT_DEFER = 2 };
constexpr uint32_t kDeferCap = 1u << 16;  // words per ring half; two halves per CTA (overflow -> L2)

struct Spill {
  uint32_t pnr;    // P * R: words >= pnr are invalid
  Div dv;
  int32_t* H;
  uint32_t* cnt;   // shared: positions handed out in this ring half so far (monotone, wraps mod 2^32)
  uint32_t* ring;  // the ring half of the current tile (kDeferCap words)
  uint32_t base;   // its first position not yet consumed; appends stay below base + kDeferCap
};

__device__ __forceinline__ void red_bin(uint32_t w, const Spill& S) { atomicAdd(S.H + hidx(w, S.dv), 1); }

// warp-aggregated append of the lanes with `mine` (all lanes of `am` call this together)
__device__ __forceinline__ void defer_warp(uint32_t am, bool mine, uint32_t w, const Spill& S) {
  const uint32_t m = __ballot_sync(am, mine);
  if (!m) return;
  const uint32_t lane = threadIdx.x & 31u, lead = __ffs(m) - 1;
  uint32_t p = 0;
  if (lane == lead) p = atomicAdd(S.cnt, (uint32_t)__popc(m));
  p = __shfl_sync(am, p, lead) + __popc(m & ((1u << lane) - 1u));
  if (mine) {
    if (p - S.base < kDeferCap) S.ring[p & (kDeferCap - 1)] = w;
    else red_bin(w, S);  // ring full: straight to L2
  }
}

// the rare part of a batch: outside the window (or invalid), or a 16-bit half that needs draining
template <int OUT>
__device__ __forceinline__ void out_of_window(uint32_t am, bool out, uint32_t w, const Spill& S, uint32_t& bad) {
#if defined(GS_DIAG) && GS_DIAG == 5  // diagnostic: deferred samples dropped
  if (OUT == OUT_DEFER) return;
#endif
#if defined(GS_DIAG) && GS_DIAG == 7  // diagnostic: n_invalid reports the deferred samples
  if (OUT == OUT_DEFER) { if (out) bad++; return; }
#endif
#if defined(GS_DIAG) && GS_DIAG == 8  // diagnostic: n_invalid reports the samples sent to L2
  if (OUT == OUT_RED) { if (out) bad++; return; }
#endif
  if (OUT == OUT_DEFER) defer_warp(am, out && w < S.pnr, w, S);
  if (out) {
    if (w >= S.pnr) bad++;
    else if (OUT == OUT_RED) red_bin(w, S);
  }
}

// 16-bit drain (out of line): the half of tab[idx] selected by sh was already >= 0x8000
__device__ __noinline__ void drain16(uint32_t* tab, uint32_t idx, uint32_t sh, uint32_t w, Div dv, int32_t* H) {
  uint32_t v = tab[idx];
  while ((v >> sh) & 0x8000u) {  // several threads may race; each successful CAS moves exactly 0x8000
    const uint32_t prev = atomicCAS(tab + idx, v, v - (0x8000u << sh));
    if (prev == v) {
      atomicAdd(H + hidx(w, dv), 0x8000);
      return;
    }
    v = prev;
  }
}

template <int OUT, int N>
__device__ __forceinline__ void count32(const uint32_t (&w)[N], Win W, uint32_t* tab, uint32_t spare, uint32_t one,
                                        const Spill& S, uint32_t& bad) {
  bool all_in = true;
#pragma unroll
  for (int q = 0; q < N; q++) {
    const uint32_t off = w[q] - W.wb;
    const bool in = off < W.lim;
    atomicAdd(tab + (in ? off : spare), one);  // the lane's spare word is never flushed
    all_in &= in;
  }
  const uint32_t am = __activemask();
  if (!__all_sync(am, all_in)) {
#pragma unroll
    for (int q = 0; q < N; q++) out_of_window<OUT>(am, w[q] - W.wb >= W.lim, w[q], S, bad);
  }
}

template <int OUT, int N>
__device__ __forceinline__ void count16(const uint32_t (&w)[N], Win W, uint32_t* tab, uint32_t spare, uint32_t one,
                                        const Spill& S, uint32_t& bad) {
  // Per sample: off, in, word, half increment, one returning shared atomic, one mask test. A lane
  // outside the window adds 2 to its spare word (never flushed; initialised to 1, so it stays odd
  // and can never wrap to 0) and its mask is all ones, so the same test flags "outside the window"
  // and "half already >= 0x8000". One vote per
  // batch; the rare path re-reads the words to find the halves to drain. Every thread that sees
  // a half >= 0x8000 checks it before its next batch, so a half overshoots 0x8000 by at most
  // (threads x batch) < 0x8000 increments before it is drained.
  uint32_t flag = 0;
#pragma unroll
  for (int q = 0; q < N; q++) {
    const uint32_t off = w[q] - W.wb;
    const bool in = off < W.lim;
    const uint32_t inc = one << ((off & 1u) << 4);
    flag |= atomicAdd(tab + (in ? off >> 1 : spare), in ? inc : 2u) & (in ? inc << 15 : 0xffffffffu);
  }
  const uint32_t am = __activemask();
  if (__any_sync(am, flag)) {
#pragma unroll
    for (int q = 0; q < N; q++) {
      const uint32_t off = w[q] - W.wb;
      out_of_window<OUT>(am, off >= W.lim, w[q], S, bad);
      if (flag && off < W.lim && ((tab[off >> 1] >> ((off & 1u) << 4)) & 0x8000u))
        drain16(tab, off >> 1, (off & 1u) << 4, w[q], S.dv, S.H);
    }
  }
}

// flush the window's counters into H and zero them (bin i of the window <-> slot ws + i / R,
// reason i % R); P16: word i holds bins 2i (low half) and 2i + 1 (high half)
template <bool P16>
__device__ void flush(uint32_t* tab, uint32_t ws, uint32_t nr, uint32_t row, uint32_t nbins, int32_t* H, uint32_t t,
                      uint32_t nt) {
  if (P16 && row == nr && ((ws * nr) & 1u) == 0 && (reinterpret_cast<uintptr_t>(H) & 7u) == 0) {
    // compact rows: the two bins of word i are adjacent int32 of H (window-relative bins 2i, 2i+1
    // at H[ws*R + 2i], 8-byte aligned), so one 64-bit L2 atomic adds both halves. Exact: bins stay
    // below 2^31, so the low word never carries into the high one.
    unsigned long long* H2 = reinterpret_cast<unsigned long long*>(H + (uint64_t)ws * nr);
    for (uint32_t i = t; 2 * i < nbins; i += nt) {
      const uint32_t v = tab[i];
      if (v) {
        tab[i] = 0;
        if (2 * i + 1 < nbins) atomicAdd(H2 + i, (unsigned long long)(v & 0xffffu) | ((unsigned long long)(v >> 16) << 32));
        else atomicAdd(H + (uint64_t)ws * nr + 2 * i, (int32_t)(v & 0xffffu));  // last, unpaired bin
      }
    }
    return;
  }
  const uint32_t per = P16 ? 2u : 1u;
  const uint32_t stride = per * nt, step_q = stride / nr, step_r = stride % nr;
  uint32_t q = (per * t) / nr, r = (per * t) % nr;
  for (uint32_t i = t; per * i < nbins; i += nt) {
    const uint32_t v = tab[i];
#if defined(GS_DIAG) && GS_DIAG == 6  // diagnostic: flush only zeroes
    tab[i] = 0;
    continue;
#endif
    if (v) {
      tab[i] = 0;
      if (!P16) {
        atomicAdd(H + (uint64_t)(ws + q) * row + r, (int32_t)v);
      } else {
        if (v & 0xffffu) atomicAdd(H + (uint64_t)(ws + q) * row + r, (int32_t)(v & 0xffffu));
        if (v >> 16) {
          const uint32_t q1 = r + 1 == nr ? q + 1 : q, r1 = r + 1 == nr ? 0 : r + 1;
          atomicAdd(H + (uint64_t)(ws + q1) * row + r1, (int32_t)(v >> 16));
        }
      }
    }
    q += step_q;
    r += step_r;
    if (r >= nr) { r -= nr; q++; }
  }
}

// Tile queue of the WINDOW kernel. Chunk c (CTA c's contiguous share) is cut into tiles of kTile4
// uint4; rng[c] = (head << 32) | stolen counts tiles taken from the front by the owner and from the
// back by CTAs that finished their own chunk (work stealing: every SM stays busy to the end while
// each CTA still walks its own chunk front to back, so windows change rarely).
// chunk c of the stream = uint4 range [bnd[c], bnd[c + 1]) (k_plan balances the chunks' cost)
__device__ __forceinline__ uint32_t n_tiles(uint64_t c, const unsigned long long* __restrict__ bnd) {
  const uint64_t a4 = bnd[c], e4 = bnd[c + 1];
  return e4 > a4 ? (uint32_t)((e4 - a4 + kTile4 - 1) / kTile4) : 0u;
}
// Called by the whole producer warp (result broadcast). Own chunk: lane 0 takes the next tile from
// the front. Stealing: the 32 lanes read the queue words of all chunks in parallel (a serial scan
// by one lane took longer than the tiles it was meant to rebalance), pick the chunk with the most
// tiles left and take its last tile with one CAS.
__device__ unsigned long long grab_tile(unsigned long long* rng, uint32_t me, uint32_t grid,
                                        const unsigned long long* __restrict__ bnd) {
  const uint32_t lane = threadIdx.x & 31u;
  unsigned long long got = ~0ull;
  if (lane == 0) {
    const uint32_t mine = n_tiles(me, bnd);
    for (;;) {  // own chunk, front to back
      const unsigned long long o = *(volatile unsigned long long*)(rng + me);
      const uint32_t head = (uint32_t)(o >> 32), stolen = (uint32_t)o;
      if (head + stolen >= mine) break;
      if (atomicCAS(rng + me, o, o + (1ull << 32)) == o) { got = ((unsigned long long)me << 32) | head; break; }
    }
  }
  got = __shfl_sync(0xffffffffu, got, 0);
  if (got != ~0ull) return got;
  for (;;) {  // steal from the back of the chunk with the most tiles left
    uint32_t best = grid, best_left = 0;
    for (uint32_t v = lane; v < grid; v += 32) {
      const unsigned long long o = *(volatile unsigned long long*)(rng + v);
      const uint32_t nt = n_tiles(v, bnd), used = (uint32_t)(o >> 32) + (uint32_t)o;
      if (nt > used && nt - used > best_left) { best_left = nt - used; best = v; }
    }
    const uint32_t mx = __reduce_max_sync(0xffffffffu, best_left);
    if (mx == 0) return ~0ull;
    const uint32_t cand = __reduce_min_sync(0xffffffffu, best_left == mx ? best : 0xffffffffu);
    if (lane == 0) {
      const unsigned long long o = *(volatile unsigned long long*)(rng + cand);
      const uint32_t nt = n_tiles(cand, bnd), head = (uint32_t)(o >> 32), stolen = (uint32_t)o;
      if (head + stolen < nt && atomicCAS(rng + cand, o, o + 1ull) == o)
        got = ((unsigned long long)cand << 32) | (nt - 1 - stolen);
    }
    got = __shfl_sync(0xffffffffu, got, 0);
    if (got != ~0ull) return got;
  }
}

// kernel of a slot: last k with kd[k].first <= slot (kernels are contiguous slot ranges, sorted)
__device__ __forceinline__ uint32_t kernel_of(uint32_t slot, const KDesc* __restrict__ kd, uint32_t nk) {
  uint32_t lo = 0, hi = nk;
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (__ldg(&kd[mid].first) <= slot) lo = mid;
    else hi = mid;
  }
  return lo;
}

// the window for a slot: its whole kernel when that fits, else nslots slots centred on it inside
// the kernel; moved down one slot when its first bin ws*R is odd (the 64-bit pair flush wants an
// even first bin; the extra slot in front is harmless, a slot lost at the end is deferred)
__device__ uint32_t window_for(uint32_t slot, const KDesc* __restrict__ kd, uint32_t nk, uint32_t nslots, uint32_t nr) {
  const KDesc K = kd[kernel_of(slot, kd, nk)];
  uint32_t ws;
  if (K.n <= nslots) {
    ws = K.first;
  } else {
    const uint32_t cws = slot > nslots / 2 ? slot - nslots / 2 : 0;
    ws = min(max(cws, K.first), K.first + K.n - nslots);
  }
  return ((ws * nr) & 1u) ? ws - 1 : ws;
}

// median slot of one valid-or-not probe per lane (~0u if no lane holds a valid word)
__device__ __forceinline__ uint32_t probe_median(bool ok, uint32_t slot) {
  uint32_t le = 0;
  for (int j = 0; j < 32; j++) le += __shfl_sync(0xffffffffu, slot, j) <= slot ? 1u : 0u;
  const uint32_t nvalid = __popc(__ballot_sync(0xffffffffu, ok));
  return __reduce_min_sync(0xffffffffu, ok && 2 * le > nvalid ? slot : 0xffffffffu);
}

// uint4 [i0, i1) of the stream, thread ct of nct: kVec 128-bit loads in flight, then the batch
template <int OUT, bool P16>
__device__ __forceinline__ void count_span(const uint4* __restrict__ s4, uint64_t i0, uint64_t i1, uint32_t ct,
                                           uint32_t nct, Win W, uint32_t* tab, uint32_t spare, uint32_t one,
                                           const Spill& S, uint32_t& bad) {
  uint64_t i = i0 + ct;
  for (; i + (kVec - 1) * nct < i1; i += kVec * nct) {
    uint32_t w[4 * kVec];
#pragma unroll
    for (int u = 0; u < kVec; u++) {
      const uint4 v = __ldg(s4 + i + u * nct);
      w[4 * u] = v.x; w[4 * u + 1] = v.y; w[4 * u + 2] = v.z; w[4 * u + 3] = v.w;
    }
    if (P16) {
      count16<OUT>(w, W, tab, spare, one, S, bad);
    } else {
      count32<OUT>(w, W, tab, spare, one, S, bad);
    }
  }
  for (; i < i1; i += nct) {
    const uint4 v = __ldg(s4 + i);
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
    if (P16) count16<OUT>(w, W, tab, spare, one, S, bad);
    else count32<OUT>(w, W, tab, spare, one, S, bad);
  }
}

// ring positions [b, b + nd) of one half, all threads, 16 loads in flight; what falls outside the
// window goes to L2. Padding lanes read an invalid word, counted as invalid and taken back out.
template <bool P16>
__device__ __forceinline__ void count_ring(const uint32_t* ring, uint32_t b, uint32_t nd, Win W, uint32_t* tab,
                                           uint32_t spare, uint32_t one, const Spill& S, uint32_t& bad, uint32_t t,
                                           uint32_t nt) {
  for (uint32_t j0 = 0; j0 < nd; j0 += 16 * nt) {
    uint32_t w[16], pad = 0;
#pragma unroll
    for (int u = 0; u < 16; u++) {
      const uint32_t j = j0 + u * nt + t;
      w[u] = j < nd ? ring[(b + j) & (kDeferCap - 1)] : 0xffffffffu;
      pad += j < nd ? 0u : 1u;
    }
#pragma unroll
    for (int u = 0; u < 4; u++) {
      const uint32_t wq[4] = {w[4 * u], w[4 * u + 1], w[4 * u + 2], w[4 * u + 3]};
      if (P16) count16<OUT_RED>(wq, W, tab, spare, one, S, bad);
      else count32<OUT_RED>(wq, W, tab, spare, one, S, bad);
    }
    bad -= pad;
  }
}

// ---------------------------------------------------------------------- WINDOW counting loop
// The hot loop keeps only the stream position, the window and the table live: everything the rare
// path needs (deferral ring, histogram, divisor) is read from shared memory / re-loaded inside the
// out-of-line rare_w, so that ptxas can issue all kVec 128-bit loads of a batch before its first
// atomic (with the rare state live, it delayed the last load behind the atomics, exposing the HBM
// latency twice per batch).
constexpr uint32_t kNct = kThreads - 32;  // counting threads of the WINDOW kernel
// 16-bit exactness: after a half reaches 0x8000 every counting thread adds at most one batch
// (4 * kVec samples) before it drains it, so the half stays below 0x10000
static_assert(kNct * 4 * kVec < 0x8000, "16-bit counters: too many increments in flight");

// the rare part of one batch of nv uint4 at s4[i + u * kNct], re-read from L1/L2: outside the
// window (deferred / invalid), or a 16-bit half that needs draining. Returns the invalid count.
// Hot words of an item (skew, e.g. C5: 90% of the samples on 10 PCs): samples equal to one of them
// are counted in registers and added to H once per item, instead of hammering one shared counter
// with same-address atomics (the north star's warp aggregation, for the case where it pays).
struct Hot {
  uint32_t w[3];  // the first n are hot words (every 32-bit value is a possible sample word: no sentinel)
  uint32_t n;
};
__device__ __forceinline__ bool is_hot(uint32_t x, const Hot& h) {
  return (h.n > 0 && x == h.w[0]) || (h.n > 1 && x == h.w[1]) || (h.n > 2 && x == h.w[2]);
}

template <bool P16, uint32_t NCT>
__device__ __noinline__ uint32_t rare_w(const uint4* __restrict__ s4, uint64_t i, uint32_t nv, Win W, uint32_t* tab,
                                        uint32_t flag, uint32_t am, const Spill S, Hot hot) {
  // (S by value: with the pointer, nvcc specialised the call to the one shared-memory state of its
  // single caller and the WINDOW kernel's register allocation came out 4% slower on C4)
  uint32_t bad = 0;
  for (uint32_t u = 0; u < nv; u++) {
    const uint4 v = __ldg(s4 + i + (uint64_t)u * NCT);
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int q = 0; q < 4; q++) {
      const uint32_t off = is_hot(w[q], hot) ? 0u : w[q] - W.wb;  // hot words: counted in registers
      const bool hw = is_hot(w[q], hot);
      out_of_window<OUT_DEFER>(am, !hw && off >= W.lim, w[q], S, bad);
      if (P16 && flag && !hw && off < W.lim && ((tab[off >> 1] >> ((off & 1u) << 4)) & 0x8000u))
        drain16(tab, off >> 1, (off & 1u) << 4, w[q], S.dv, S.H);
    }
  }
  return bad;
}

// the sample stream is read once: evict-first loads keep L2 for the histogram the flushes update
// (bench context, same box: 0.790 -> 0.777 ms after detect + rank; GS_NO_LDCS: plain __ldg)
#ifndef GS_NO_LDCS
__device__ __forceinline__ uint4 ld_stream(const uint4* p) { return __ldcs(p); }
#else
__device__ __forceinline__ uint4 ld_stream(const uint4* p) { return __ldg(p); }
#endif

// per-sample fast path of one batch; returns the lane's flag (nonzero: rare work in this batch)
template <bool P16, int N>
__device__ __forceinline__ uint32_t hot_w(const uint32_t (&w)[N], Win W, uint32_t* tab, uint32_t spare) {
  uint32_t flag = 0;
#pragma unroll
  for (int q = 0; q < N; q++) {
    const uint32_t off = w[q] - W.wb;
    const bool in = off < W.lim;
    if (P16) {
      const uint32_t inc = 1u << ((off & 1u) << 4);  // spare word: +2 keeps it odd (nonzero)
      flag |= atomicAdd(tab + (in ? off >> 1 : spare), in ? inc : 2u) & (in ? inc << 15 : 0xffffffffu);
    } else {
      atomicAdd(tab + (in ? off : spare), 1u);
      flag |= in ? 0u : 1u;
    }
  }
  return flag;
}

// shared-memory atomic add executed only when p (a predicated ATOMS, no branch); 0 otherwise
__device__ __forceinline__ uint32_t atoms_add_if(bool p, uint32_t* addr, uint32_t v) {
  uint32_t r = 0;
  asm volatile(
      "{\n .reg .pred q;\n setp.ne.u32 q, %3, 0;\n @q atom.shared.add.u32 %0, [%1], %2;\n}"
      : "+r"(r)
      : "r"((uint32_t)__cvta_generic_to_shared(addr)), "r"(v), "r"(p ? 1u : 0u)
      : "memory");
  return r;
}

// the fast path with hot words: a hot sample adds to its register counter and issues no atomic
template <bool P16, int N>
__device__ __forceinline__ uint32_t hot_w_skew(const uint32_t (&w)[N], Win W, uint32_t* tab, uint32_t spare,
                                               const Hot& h, uint32_t& c) {
  uint32_t flag = 0;
#pragma unroll
  for (int q = 0; q < N; q++) {
    const bool m0 = h.n > 0 && w[q] == h.w[0], m1 = h.n > 1 && w[q] == h.w[1], m2 = h.n > 2 && w[q] == h.w[2];
    c += (m0 ? 1u : 0u) + (m1 ? 1u << 10 : 0u) + (m2 ? 1u << 20 : 0u);  // three 10-bit counters, one register
    const bool cold = !(m0 | m1 | m2);
    const uint32_t off = w[q] - W.wb;
    const bool in = off < W.lim;
    if (P16) {
      const uint32_t inc = 1u << ((off & 1u) << 4);
      flag |= atoms_add_if(cold, tab + (in ? off >> 1 : spare), in ? inc : 2u) & (in ? inc << 15 : 0xffffffffu);
    } else {
      atoms_add_if(cold, tab + (in ? off : spare), 1u);
      flag |= (cold && !in) ? 1u : 0u;
    }
  }
  return flag;
}

template <bool P16, uint32_t NCT = kNct, bool HOT = false>
__device__ __forceinline__ uint32_t count_span_w(const uint4* __restrict__ s4, uint64_t i0, uint64_t i1, uint32_t ct,
                                                 Win W, uint32_t* tab, uint32_t spare, const Spill* sS,
                                                 Hot hot = Hot{{0u, 0u, 0u}, 0u}) {
  uint32_t bad = 0, c = 0;  // HOT: packed counters of the 3 hot words (< 1024 per item and thread)
  uint64_t i = i0 + ct;
  for (; i + (kVec - 1) * NCT < i1; i += kVec * NCT) {
    uint32_t w[4 * kVec];
#pragma unroll
    for (int u = 0; u < kVec; u++) {
      const uint4 v = ld_stream(s4 + i + u * NCT);
      w[4 * u] = v.x; w[4 * u + 1] = v.y; w[4 * u + 2] = v.z; w[4 * u + 3] = v.w;
    }
    const uint32_t flag = HOT ? hot_w_skew<P16>(w, W, tab, spare, hot, c) : hot_w<P16>(w, W, tab, spare);
    const uint32_t am = __activemask();
    if (__any_sync(am, flag)) bad += rare_w<P16, NCT>(s4, i, kVec, W, tab, flag, am, *sS, hot);
  }
  for (; i < i1; i += NCT) {
    const uint4 v = __ldg(s4 + i);
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
    const uint32_t flag = HOT ? hot_w_skew<P16>(w, W, tab, spare, hot, c) : hot_w<P16>(w, W, tab, spare);
    const uint32_t am = __activemask();
    if (__any_sync(am, flag)) bad += rare_w<P16, NCT>(s4, i, 1, W, tab, flag, am, *sS, hot);
  }
  if (HOT) {  // the item's hot counts, one L2 reduction per hot word and thread
    const Spill S = *sS;
#pragma unroll
    for (int j = 0; j < 3; j++) {
      const uint32_t cj = (c >> (10 * j)) & 1023u;
      if (cj && (uint32_t)j < hot.n) atomicAdd(S.H + hidx(hot.w[j], S.dv), (int32_t)cj);
    }
  }
  return bad;
}

// ---------------------------------------------------------------------- PRIVATE
// fixed slot range per CTA (range = blockIdx % n_ranges); the CTA walks its sample chunk.
// 16-bit exactness (count16): the increment that takes a half from 0x7FFF to 0x8000 is not flagged,
// every later one is, and a thread drains at the end of its batch. In the worst case every one of
// the kThreads threads adds a whole batch (4 * kVec samples) to the half after it reached 0x8000
// and before any drain, so the half peaks at 0x7FFF + kThreads * 4 * kVec: at most 0xFFFF, never a
// carry into the neighbouring bin, iff kThreads * 4 * kVec <= 0x8000.
static_assert(kThreads * 4 * kVec <= 0x8000, "PRIVATE 16-bit counters: a half could carry into its neighbour");
template <bool P16>
__global__ void __launch_bounds__(kThreads, 1)
    k_hist_smem(const uint32_t* __restrict__ s, uint64_t n, uint32_t P, uint32_t nr, Div dv, uint32_t n_ranges,
                uint64_t chunk, uint32_t one, int32_t* __restrict__ H, unsigned long long* d_n_invalid) {
  extern __shared__ uint32_t tab[];
  const uint32_t pnr = P * nr;
  const uint32_t nslots = (P16 ? 2 * kTableWords : kTableWords) / nr;
  const uint32_t spare = kTableWords + (threadIdx.x & 31u);
  const uint32_t range = blockIdx.x % n_ranges;
  const uint64_t ci = blockIdx.x / n_ranges;
  const uint32_t ws = range * nslots;
  const Win W{ws * nr, min(nslots, P - min(P, ws)) * nr};
  for (uint32_t i = threadIdx.x; i < kTableWords + 32; i += blockDim.x) tab[i] = i < kTableWords ? 0u : 1u;
  uint32_t bad = 0;
  const Spill S{pnr, dv, H, nullptr, nullptr, 0};
  __syncthreads();
  const uint64_t e_own = (ci + 1) * chunk < n ? (ci + 1) * chunk : n;
  count_span<OUT_DROP, P16>(reinterpret_cast<const uint4*>(s), ci * chunk / 4, e_own / 4, threadIdx.x, blockDim.x, W,
                            tab, spare, one, S, bad);
  // the last chunk's words after its last 16-byte boundary (< 4 words): L2 atomics
  if (e_own == n && range == 0)
    for (uint64_t i = e_own / 4 * 4 + threadIdx.x; i < n; i += blockDim.x) {
      if (s[i] < pnr) atomicAdd(H + hidx(s[i], dv), 1);
      else bad++;
    }
  if (range == 0) count_invalid(bad, d_n_invalid);
  __syncthreads();
  flush<P16>(tab, ws, nr, dv.row, W.lim, H, threadIdx.x, blockDim.x);
}

// ---------------------------------------------------------------------- WINDOW
__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {  // release.cta
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {  // acquire.cta
  asm volatile(
      "{\n .reg .pred p;\n WAIT%=:\n mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n @!p bra WAIT%=;\n}" ::"r"(
          smem_u32(bar)),
      "r"(parity)
      : "memory");
}
// the producer's wait for a free item slot: back off between polls so that the spinning warp
// does not take shared-memory cycles from the counters' atomics
__device__ __forceinline__ void mbar_wait_backoff(uint64_t* bar, uint32_t parity) {
  uint32_t ok = 0;
  for (;;) {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n selp.u32 %0, 1, 0, p;\n}"
        : "=r"(ok)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
    if (ok) return;
#ifndef GS_BACKOFF_NS
#define GS_BACKOFF_NS 500
#endif
    if (GS_BACKOFF_NS) __nanosleep(GS_BACKOFF_NS);
  }
}
// the 31 counting warps only (warp 0 keeps producing)
__device__ __forceinline__ void bar_counters() { asm volatile("bar.sync 1, %0;" ::"r"(kThreads - 32) : "memory"); }

#ifndef GS_ITEMS
#define GS_ITEMS 8
#endif
constexpr uint32_t kItems = GS_ITEMS;  // descriptor ring depth
struct Item {
  uint64_t a4, b4;  // uint4 range of the stream
  uint32_t ws;      // window (first slot) for the range
  uint32_t last;    // 1: no more work
  Hot hot;          // hot words of the tile (hot.n of them)
};
// a probe word seen in at least kHotMin of the tile's 32 probes is a hot word of the tile
#ifndef GS_HOT_MIN
#define GS_HOT_MIN 3
#endif

// One persistent CTA per SM. Warp 0 (producer) grabs tiles from the work-stealing queue, picks
// each tile's window(s) from 32 probe samples and publishes (range, window) items through an
// mbarrier ring; warps 1..31 (counters) count each item into the shared table. The counters only
// synchronise with each other when the window changes (named barrier, flush, barrier), so tiles
// can be small (short tail) without a CTA-wide barrier per tile.
//
// Window choice per tile (lane j probes position j/32 of the tile):
//  * the probes' kernels form two runs (the tile crosses from one kernel launch into the next, as
//    a PC-sampling trace does): two items split at the first probe of the second run, each with
//    the window of its own probes;
//  * otherwise one item with one window.
// A part keeps the previous window when that holds all of its valid probes (a large kernel's
// window re-centres when the median nears its edge); else the window of its probes' median.
// Samples outside the window in force go to the CTA's deferral ring (half = epoch & 1, an epoch
// being a run of items with one window) and are counted right after the next window switch,
// against the new window (a straddling tile's early samples of the next kernel land there).
template <bool P16>
__global__ void __launch_bounds__(kThreads, 1)
    k_hist_window(const uint32_t* __restrict__ s, uint64_t n, uint32_t P, uint32_t nr, Div dv,
                  const KDesc* __restrict__ kd, uint32_t nk, uint32_t one, int32_t* __restrict__ H,
                  unsigned long long* d_n_invalid, unsigned long long* rng, uint32_t* __restrict__ defer_ring,
                  uint32_t tw) {
  const unsigned long long* __restrict__ bnd = rng + gridDim.x;  // chunk bounds (k_plan)
  extern __shared__ uint32_t tab[];  // tw counter words + 32 spare words
  __shared__ Item items[kItems];
  __shared__ __align__(8) uint64_t full[kItems], empty[kItems];
  __shared__ uint32_t sh_ndefer[2];
  __shared__ Spill sh_S;  // the counters' rare-path state (written at window switches)
  const uint32_t pnr = P * nr;
  const uint32_t nslots = (P16 ? 2 * tw : tw) / nr;
  const uint32_t lane = threadIdx.x & 31u;
  for (uint32_t i = threadIdx.x; i < tw + 32; i += blockDim.x) tab[i] = i < tw ? 0u : 1u;
  if (threadIdx.x < kItems) {
    mbar_init(&full[threadIdx.x], 1);
    mbar_init(&empty[threadIdx.x], kThreads / 32 - 1);
  }
  if (threadIdx.x < 2) sh_ndefer[threadIdx.x] = 0;
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  __syncthreads();

  const auto span = [&](unsigned long long tile, uint64_t& a4, uint64_t& b4) {
    const uint64_t c = tile >> 32, ce4 = bnd[c + 1];
    a4 = bnd[c] + (uint64_t)(uint32_t)tile * kTile4;
    b4 = a4 + kTile4 < ce4 ? a4 + kTile4 : ce4;
  };

  if (threadIdx.x < 32) {  // ------------------------------------------------ producer
    uint32_t pws = kNoWindow, j = 0;
    Hot hot{{0u, 0u, 0u}, 0u};
    const auto publish = [&](uint64_t a4, uint64_t b4, uint32_t ws, uint32_t last) {
      const uint32_t k = j % kItems;
      if (lane == 0) {
        mbar_wait_backoff(&empty[k], ((j / kItems) & 1u) ^ 1u);
        items[k] = Item{a4, b4, ws, last, hot};
        mbar_arrive(&full[k]);
      }
      __syncwarp();
      j++;
    };
    for (;;) {
      const unsigned long long tile = grab_tile(rng, blockIdx.x, gridDim.x, bnd);
      if (tile == ~0ull) break;
      uint64_t a4, b4;
      span(tile, a4, b4);
      const uint64_t at4 = a4 + (b4 - a4) * lane / 32;
      const uint32_t w = __ldg(s + 4 * at4);
      const bool ok = w < pnr;
      const uint32_t slot = ok ? divq(w, dv) : 0xffffffffu;
      const uint32_t k = ok ? kernel_of(slot, kd, nk) : 0xffffffffu;
      const uint32_t okm = __ballot_sync(0xffffffffu, ok);
      {  // hot words: the most frequent valid probe words seen >= GS_HOT_MIN times (at most 3)
        const uint32_t mm = __match_any_sync(0xffffffffu, w);
        uint32_t cnt = (ok && (uint32_t)(__ffs(mm) - 1) == lane) ? (uint32_t)__popc(mm) : 0u;
        hot.n = 0;
#pragma unroll
        for (int q = 0; q < 3; q++) {
          const uint32_t key = cnt >= GS_HOT_MIN ? (cnt << 5) | lane : 0u;
          const uint32_t best = __reduce_max_sync(0xffffffffu, key);
          const uint32_t bl = best & 31u;
          const uint32_t bw = __shfl_sync(0xffffffffu, w, bl);
          hot.w[q] = bw;
          hot.n += best ? 1u : 0u;  // keys are taken in decreasing order: the hot words come first
          if (best && lane == bl) cnt = 0;
        }
      }
      const uint32_t k0 = __reduce_min_sync(0xffffffffu, k), k1 = __reduce_max_sync(0xffffffffu, ok ? k : 0u);
      const uint32_t m0 = __ballot_sync(0xffffffffu, ok && k == k0), m1 = __ballot_sync(0xffffffffu, ok && k == k1);
      // one window for the probes of mask pm, given the window before them
      const auto pick = [&](uint32_t pm, uint32_t cur) {
        const bool mine = (pm >> lane) & 1u;
        const uint32_t outm = __ballot_sync(0xffffffffu, mine && (cur == kNoWindow || slot - cur >= nslots));
        const uint32_t med = probe_median(mine, slot);
        if (med == 0xffffffffu) return cur == kNoWindow ? 0u : cur;
        if (!outm && med - cur >= nslots / 8 && med - cur < nslots - nslots / 8) return cur;
        return window_for(med, kd, nk, nslots, nr);
      };
      // two runs: valid probes all in k0 or k1 (k0 != k1), every k0 probe before every k1 probe
      const bool two_runs = okm && k0 != k1 && (m0 | m1) == okm && 31 - __clz(m0) < __ffs(m1) - 1;
      if (two_runs) {
        const uint32_t ws1 = pick(m0, pws), ws2 = pick(m1, ws1);
        if (ws2 != ws1) {
          const uint64_t mid = __shfl_sync(0xffffffffu, at4, __ffs(m1) - 1);
          publish(a4, mid, ws1, 0);
          publish(mid, b4, ws2, 0);
        } else {
          publish(a4, b4, ws1, 0);
        }
        pws = ws2;
      } else {
        pws = pick(okm, pws);
        publish(a4, b4, pws, 0);
      }
    }
    publish(0, 0, pws, 1);
    return;
  }

  // --------------------------------------------------------------------------- counters
  const uint32_t ct = threadIdx.x - 32, nct = kThreads - 32;
  const uint32_t spare = tw + lane;
  const uint4* s4 = reinterpret_cast<const uint4*>(s);
  uint32_t* const ring0 = defer_ring + (uint64_t)blockIdx.x * 2 * kDeferCap;
  uint32_t bad = 0, ws = kNoWindow, epoch = 0, dstart0 = 0, dstart1 = 0;
  Win W{0, 0};
  Spill S{pnr, dv, H, &sh_ndefer[0], ring0, 0};
#if defined(GS_DIAG) && GS_DIAG == 11  // diagnostic: per-CTA timeline (printf)
  long long d_t0 = clock64(), d_wait = 0, d_flush = 0, d_ring = 0, d_count = 0;
  uint32_t d_sw = 0, d_items = 0;
  uint64_t d_words = 0;
#define GS_T(acc, ...) { const long long _a = clock64(); __VA_ARGS__; acc += clock64() - _a; }
#else
#define GS_T(acc, ...) { __VA_ARGS__; }
#endif
  for (uint32_t j = 0;; j++) {
    const uint32_t k = j % kItems;
    GS_T(d_wait, mbar_wait(&full[k], (j / kItems) & 1u));
    const Item it = items[k];
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[k]);
    if (it.last) break;
#if defined(GS_DIAG) && GS_DIAG == 10  // diagnostic: n_invalid counts items
    if (ct == 0) atomicAdd(d_n_invalid, 1ull);
#endif
    if (it.ws != ws) {  // window switch: every counter is done with the old window
#if defined(GS_DIAG) && GS_DIAG == 9  // diagnostic: n_invalid counts window switches
      if (ct == 0) atomicAdd(d_n_invalid, 1ull);
#endif
      GS_T(d_flush, bar_counters(); if (ws != kNoWindow) flush<P16>(tab, ws, nr, dv.row, W.lim, H, ct, nct);
           bar_counters());
#if defined(GS_DIAG) && GS_DIAG == 11
      d_sw++;
#endif
      ws = it.ws;
      W = Win{ws * nr, min(nslots, P - min(P, ws)) * nr};
      if (ws != kNoWindow && j) {  // the ended epoch's deferred samples, against the new window
        const uint32_t h = epoch & 1u, dend = sh_ndefer[h], db = h ? dstart1 : dstart0;
        if (dend != db)  // positions past the capacity went to L2 when they were deferred
          GS_T(d_ring, count_ring<P16>(ring0 + h * kDeferCap, db, min(dend - db, kDeferCap), W, tab, spare, one, S, bad, ct, nct));
        if (h) dstart1 = dend;
        else dstart0 = dend;
        epoch++;
      }
      const uint32_t h = epoch & 1u;  // the new epoch appends to the other half
      S.cnt = &sh_ndefer[h];
      S.ring = ring0 + h * kDeferCap;
      S.base = h ? dstart1 : dstart0;
      if (ct == 0) sh_S = S;
      bar_counters();
    }
    if (it.hot.n) {
      GS_T(d_count, bad += count_span_w<P16, kNct, true>(s4, it.a4, it.b4, ct, W, tab, spare, &sh_S, it.hot));
    } else {
      GS_T(d_count, bad += count_span_w<P16>(s4, it.a4, it.b4, ct, W, tab, spare, &sh_S));
    }
#if defined(GS_DIAG) && GS_DIAG == 11
    d_items++;
    d_words += 4 * (it.b4 - it.a4);
#endif
  }
  bar_counters();
  {  // the last epoch's deferred samples: what is not in the current window goes to L2
    const uint32_t h = epoch & 1u, dend = sh_ndefer[h], db = h ? dstart1 : dstart0;
    if (dend != db)
      count_ring<P16>(ring0 + h * kDeferCap, db, min(dend - db, kDeferCap), W, tab, spare, one, S, bad, ct, nct);
  }
  // the stream's words after its last 16-byte boundary (< 4 words): L2 atomics
  if (blockIdx.x == gridDim.x - 1)
    for (uint64_t i = n / 4 * 4 + ct; i < n; i += nct) {
      if (s[i] < pnr) atomicAdd(H + hidx(s[i], dv), 1);
      else bad++;
    }
  count_invalid(bad, d_n_invalid);
  long long d_f0 = clock64();
  bar_counters();
  if (ws != kNoWindow) flush<P16>(tab, ws, nr, dv.row, W.lim, H, ct, nct);
#if defined(GS_DIAG) && GS_DIAG == 11
  bar_counters();
  if (ct == 0)
    printf("DIAG11 cta %u sm_clk total %lld wait %lld flush %lld ring %lld count %lld final_flush %lld switches %u items %u words %llu\n",
           blockIdx.x, clock64() - d_t0, d_wait, d_flush, d_ring, d_count, clock64() - d_f0, d_sw, d_items,
           (unsigned long long)d_words);
#else
  (void)d_f0;
#endif
}

// Chunk planning for WINDOW: the CTAs' contiguous chunks are cut at equal COST, not at equal
// sample counts. A chunk costs its samples plus, per window switch, the flush of a whole window
// (~15K SM cycles ~ kSwitchCost samples at the counting rate): Zipf-distributed kernel weights put
// many small kernels (many switches) into the last chunks of a trace, which otherwise finish last
// (per-CTA timeline, GS_DIAG=11). kPlanProbes probe samples estimate where the windows change;
// the queue words are zeroed here too.
#ifndef GS_SWITCH_COST
#define GS_SWITCH_COST 160000
#endif
constexpr uint32_t kPlanProbes = 4096;
__global__ void __launch_bounds__(1024) k_plan(const uint32_t* __restrict__ s, uint64_t n, uint32_t pnr, Div dv,
                                               uint32_t nslots, uint32_t chunks, unsigned long long* __restrict__ q,
                                               int32_t* __restrict__ zero_h, uint64_t zero_n) {
  __shared__ unsigned long long pre[kPlanProbes];
  __shared__ unsigned long long wsum[32];
  // the histogram's zeroing (instead of a separate memset node): CTAs 1.. zero grid-strided shares
  // with 128-bit stores while CTA 0 plans (zeroing, then planning, in CTA 0 put the plan on the
  // critical path: C4 attribution 0.760 -> 0.753 ms); zero_h is 16-byte aligned, zero_n words
  if (zero_h && (blockIdx.x != 0 || gridDim.x == 1)) {
    const uint32_t zc = gridDim.x > 1 ? blockIdx.x - 1 : 0u, nzc = gridDim.x > 1 ? gridDim.x - 1 : 1u;
    uint4* h4 = reinterpret_cast<uint4*>(zero_h);
    const uint64_t n4w = zero_n / 4;
    for (uint64_t i = zc * (uint64_t)blockDim.x + threadIdx.x; i < n4w; i += (uint64_t)nzc * blockDim.x)
      h4[i] = make_uint4(0, 0, 0, 0);
    if (zc == nzc - 1 && threadIdx.x < (zero_n & 3)) zero_h[n4w * 4 + threadIdx.x] = 0;
  }
  if (blockIdx.x != 0) return;
  const uint64_t n4 = n / 4;
  const uint32_t t = threadIdx.x;
#ifdef GS_PLAN_UNIFORM  // diagnostic: equal-sample chunks (the cost of the probes)
  for (uint32_t c = t; c <= chunks; c += blockDim.x) {
    if (c < chunks) q[c] = 0ull;
    q[chunks + c] = (uint64_t)c * n4 / chunks;
  }
  return;
#endif
  constexpr uint32_t kPer = kPlanProbes / 1024;
  // probe p sits at uint4 position pos(p) = p * n4 / NP; interval p = [pos(p), pos(p + 1))
  uint32_t win[kPer + 1];
#pragma unroll
  for (uint32_t u = 0; u <= kPer; u++) {
    const uint64_t p = (uint64_t)t * kPer + u;
    const uint64_t pos = p * n4 / kPlanProbes;
    const uint32_t w = (p < kPlanProbes && pos < n4) ? __ldg(s + 4 * pos) : 0xffffffffu;
    win[u] = w < pnr ? divq(w, dv) / nslots : 0xffffffffu;  // window-sized slot block of the probe
  }
  unsigned long long loc = 0;
  unsigned long long cst[kPer];
#pragma unroll
  for (uint32_t u = 0; u < kPer; u++) {
    const uint64_t p = (uint64_t)t * kPer + u;
    const uint64_t a = p * n4 / kPlanProbes, b = (p + 1) * n4 / kPlanProbes;
    const bool sw = win[u] != 0xffffffffu && win[u + 1] != 0xffffffffu && win[u] != win[u + 1];
    cst[u] = 4 * (b - a) + (sw ? (unsigned long long)GS_SWITCH_COST : 0ull);
    loc += cst[u];
  }
  // inclusive scan of the per-thread sums over the CTA
  const uint32_t lane = t & 31u, warp = t >> 5;
  unsigned long long v = loc;
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long x = __shfl_up_sync(0xffffffffu, v, o);
    if ((int)lane >= o) v += x;
  }
  if (lane == 31) wsum[warp] = v;
  __syncthreads();
  if (warp == 0) {
    unsigned long long x = wsum[lane];
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(0xffffffffu, x, o);
      if ((int)lane >= o) x += y;
    }
    wsum[lane] = x;
  }
  __syncthreads();
  unsigned long long run = (warp ? wsum[warp - 1] : 0ull) + v - loc;  // exclusive prefix of this thread
#pragma unroll
  for (uint32_t u = 0; u < kPer; u++) {
    run += cst[u];
    pre[t * kPer + u] = run;  // cost up to the end of interval p
  }
  __syncthreads();
  const unsigned long long total = pre[kPlanProbes - 1];
  unsigned long long* bnd = q + chunks;
  for (uint32_t c = t; c <= chunks; c += blockDim.x) {
    if (c < chunks) q[c] = 0ull;
    uint64_t b;
    if (c == 0) b = 0;
    else if (c == chunks) b = n4;
    else {  // the end of the first interval whose cost prefix reaches c / chunks of the total
      const unsigned long long target = total * c / chunks;
      uint32_t lo = 0, hi = kPlanProbes - 1;
      while (lo < hi) {
        const uint32_t mid = (lo + hi) >> 1;
        if (pre[mid] >= target) hi = mid;
        else lo = mid + 1;
      }
      b = (uint64_t)(lo + 1) * n4 / kPlanProbes;
    }
    bnd[c] = b;
  }
}

// ---------------------------------------------------------------------- PARTITION
// For streams without locality (e.g. samples in random order): a WINDOW would see most samples
// outside any window (L2 atomics, ~0.12 T samples/s). Instead the samples are first partitioned by
// bucket = compact bin >> kPBits (2^kPBits bins, one shared-memory table of 32-bit counters), then
// every bucket is counted in its own table, where every sample is inside. The partitioned copy
// holds only the bin's offset inside its bucket, 16 bits per sample, so the two passes after the
// count move 4 + 2 + 2 bytes per sample instead of 4 + 4 + 4:
//   k_pcount   per CTA chunk: samples per bucket (shared counters), invalid words counted
//   k_pscan    one CTA: bucket regions (8-entry aligned starts, padding 0xFFFF) and each chunk's
//              offset per bucket
//   k_pscatter per CTA chunk, tiles of NT x 8 samples: counting sort of the tile in shared memory
//              by bucket, the 16-bit offsets written to the bucket regions (coalesced within a run)
//   k_pbucket_hist  per CTA a contiguous share of the partitioned array, bucket by bucket: one
//              non-returning shared atomic per sample, the table flushed into H at bucket switches
#ifndef GS_PBITS
#define GS_PBITS 15
#endif
constexpr uint32_t kPBits = GS_PBITS;          // bins per bucket = 2^kPBits (offsets fit 16 bits)
static_assert(kPBits <= 15, "bucket offsets are 16-bit, 0xFFFF is the padding");
constexpr uint32_t kPBins = 1u << kPBits;
constexpr uint16_t kPPad = 0xffffu;            // padding entry (>= kPBins when kPBits < 16: never counted)
constexpr int kPT = 1024;                      // threads of k_pcount / k_pscan
constexpr uint32_t kPMaxBuckets = 1024;        // B < kPMaxBuckets (+1 for the invalid words): P * R < 2^25 at kPBits = 15
constexpr uint32_t kPSub = 4;                  // rank counters per bucket (k_pscatter)
#ifndef GS_PST
#define GS_PST 1024
#endif
constexpr int kPST = GS_PST;                   // threads of k_pscatter
#ifndef GS_PV
#define GS_PV 16
#endif
constexpr uint32_t kPV = GS_PV;                // samples per thread per scatter tile
constexpr uint32_t kSTile = kPST * kPV;        // samples per scatter tile
#ifndef GS_PHT
#define GS_PHT 1024
#endif
constexpr int kPHT = GS_PHT;                   // threads of k_pbucket_hist

__device__ __forceinline__ uint32_t pbucket(uint32_t w) { return w >> kPBits; }

__global__ void __launch_bounds__(kPT) k_pcount(const uint32_t* __restrict__ s, uint64_t n, uint64_t chunk,
                                                uint32_t pnr, uint32_t B, uint32_t* __restrict__ cnt,
                                                unsigned long long* d_n_invalid) {
  __shared__ uint32_t h[kPMaxBuckets];
  for (uint32_t b = threadIdx.x; b < B; b += kPT) h[b] = 0;
  __syncthreads();
  const uint64_t a = blockIdx.x * chunk, e = min(n, a + chunk);  // chunk is a multiple of 4 words
  const uint4* s4 = reinterpret_cast<const uint4*>(s);
  uint32_t bad = 0;
  uint64_t i = a / 4 + threadIdx.x;
  const uint64_t e4 = e / 4;
  for (; i + 3 * kPT < e4; i += 4 * kPT) {
    uint4 v[4];
#pragma unroll
    for (int u = 0; u < 4; u++) v[u] = ld_stream(s4 + i + u * kPT);
#pragma unroll
    for (int u = 0; u < 4; u++) {
      const uint32_t w[4] = {v[u].x, v[u].y, v[u].z, v[u].w};
#pragma unroll
      for (int q = 0; q < 4; q++) {
        const bool ok = w[q] < pnr;
        if (ok) atomicAdd(&h[pbucket(w[q])], 1u);
        bad += ok ? 0u : 1u;
      }
    }
  }
  for (; i < e4; i += kPT) {
    const uint4 v = __ldg(s4 + i);
    const uint32_t w[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int q = 0; q < 4; q++) {
      if (w[q] < pnr) atomicAdd(&h[pbucket(w[q])], 1u);
      else bad++;
    }
  }
  for (uint64_t j = e4 * 4 + threadIdx.x; j < e; j += kPT) {  // the stream's last < 4 words
    if (s[j] < pnr) atomicAdd(&h[pbucket(s[j])], 1u);
    else bad++;
  }
  count_invalid(bad, d_n_invalid);
  __syncthreads();
  for (uint32_t b = threadIdx.x; b < B; b += kPT) cnt[(uint64_t)blockIdx.x * B + b] = h[b];
}

// bstart[b]: first entry of bucket b's region (8-aligned: whole uint4 of 16-bit entries),
// bstart[B] = end; off[c][b] = where chunk c writes its bucket-b samples (in place of cnt)
__global__ void __launch_bounds__(kPT) k_pscan(uint32_t* __restrict__ cnt, uint32_t nchunk, uint32_t B,
                                               unsigned long long* __restrict__ bstart, uint16_t* __restrict__ out) {
  __shared__ unsigned long long tot[kPMaxBuckets], pre[kPMaxBuckets];
  for (uint32_t b = threadIdx.x; b < B; b += kPT) {
    unsigned long long t = 0;
#pragma unroll 8
    for (uint32_t c = 0; c < nchunk; c++) t += cnt[(uint64_t)c * B + b];
    tot[b] = t;
  }
  __syncthreads();
  if (threadIdx.x < 32) {  // warp scan of the 8-aligned region sizes, 64 buckets per lane at most
    const uint32_t lane = threadIdx.x, per = (B + 31) / 32;
    unsigned long long sum = 0;
    for (uint32_t q = 0; q < per; q++) {
      const uint32_t b = lane * per + q;
      if (b < B) sum += (tot[b] + 7) & ~7ull;
    }
    unsigned long long inc = sum;
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += y;
    }
    unsigned long long p = inc - sum;
    for (uint32_t q = 0; q < per; q++) {
      const uint32_t b = lane * per + q;
      if (b < B) {
        pre[b] = p;
        bstart[b] = p;
        p += (tot[b] + 7) & ~7ull;
      }
    }
    if (lane == 31) bstart[B] = inc;
  }
  __syncthreads();
  for (uint32_t b = threadIdx.x; b < B; b += kPT) {
    const unsigned long long e = pre[b] + tot[b], e8 = (e + 7) & ~7ull;
    for (unsigned long long q = e; q < e8; q++) out[q] = kPPad;  // padding entries
    unsigned long long p = 0;
    for (uint32_t c = 0; c < nchunk; c++) {
      const uint32_t x = cnt[(uint64_t)c * B + b];
      cnt[(uint64_t)c * B + b] = (uint32_t)p;  // offset within the bucket (< 2^32)
      p += x;
    }
  }
}

// Counting sort of each tile of kSTile samples by bucket. The tiles of the CTA's chunk arrive in
// shared memory by TMA bulk copies (cp.async.bulk, double-buffered: the copy of tile i + 1 runs
// while tile i is sorted; no registers hold the next tile). Three barriers per tile: ranks | scan
// (resets the rank counters, advances the bucket cursors) | stage | write-out. The write-out reads
// each staged word, its bucket's destination base dst[b] = cursor - tile offset, and stores the
// 16-bit offset (consecutive threads of a run store consecutive entries).
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  if (!bytes) {  // a tile of < 4 words: nothing to copy, complete the phase
    mbar_arrive(bar);
    return;
  }
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_u32(dst)),
               "l"(src), "r"(bytes), "r"(smem_u32(bar))
               : "memory");
}
// Off: uint32_t when the partitioned array has < 2^32 entries (a 64-bit dst[] doubles the bank
// conflicts of the write-out's random lookups), else unsigned long long.
template <int NT, typename Off>
__global__ void __launch_bounds__(NT, 1) k_pscatter(const uint32_t* __restrict__ s, uint64_t n, uint64_t chunk,
                                                     uint32_t pnr, uint32_t B, const uint32_t* __restrict__ off,
                                                     const unsigned long long* __restrict__ bstart,
                                                     uint16_t* __restrict__ out) {
  // Rank counters: kPSub per bucket, lane % kPSub picks one, so lanes of a warp that hold the same
  // (Zipf-hot) bucket mostly hit different words and banks (one counter per bucket measured 6.6
  // shared-memory wavefronts per warp-level rank atomic on C4-shuffled). Thread t scans bucket t.
  static_assert(NT == kPMaxBuckets, "one bucket per scanning thread");
  __shared__ uint32_t th[kPMaxBuckets * kPSub];
  __shared__ uint16_t tcnt[kPMaxBuckets * kPSub];  // tile offset of (bucket, sub); < 2^16
  __shared__ Off dst[kPMaxBuckets];                // cursor of bucket b minus its tile offset (mod 2^bits(Off))
  __shared__ uint32_t wsum[NT / 32];
  __shared__ __align__(8) uint64_t full[2];
  constexpr uint32_t kTile = NT * kPV;  // samples per tile
  static_assert(kPV % 8 == 0, "write-out in groups of eight, uint4 reads");
  static_assert(kTile < 65536 && kPMaxBuckets * kPSub <= 65536, "packed counter/rank, 16-bit tile offsets");
  extern __shared__ __align__(16) uint32_t dyn[];    // raw[2][kTile] (TMA destinations), stage[kTile]
  uint32_t* const raw0 = dyn;
  uint32_t* const stage = dyn + 2 * kTile;
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5, sub = lane % kPSub;
  const uint32_t bt = threadIdx.x;  // the bucket this thread scans
  Off cur = bt < B ? (Off)(bstart[bt] + off[(uint64_t)blockIdx.x * B + bt]) : (Off)0;  // its cursor
  for (uint32_t i = threadIdx.x; i < (B + 1) * kPSub; i += NT) th[i] = 0;
  const uint64_t a = blockIdx.x * chunk, e = min(n, a + chunk);  // a: a multiple of kTile
  // whole 16-byte units of the tile at t0 go through TMA; the < 4 trailing words of the stream are
  // read directly
  const auto tma_words = [&](uint64_t t0) -> uint32_t { return (uint32_t)((min(e, t0 + kTile) - t0) & ~3ull); };
  if (threadIdx.x == 0) {
    mbar_init(&full[0], 1);
    mbar_init(&full[1], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    if (a < e) bulk_g2s(raw0, s + a, 4 * tma_words(a), &full[0]);
  }
  __syncthreads();
  uint32_t it = 0;
  for (uint64_t t0 = a; t0 < e; t0 += kTile, it++) {
    const uint32_t buf = it & 1u;
    const uint32_t* raw = raw0 + buf * kTile;
    if (threadIdx.x == 0 && t0 + kTile < e) {  // the next tile into the other buffer (free: every
      // thread passed barrier D of the previous tile, its last reader)
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      bulk_g2s(raw0 + (buf ^ 1u) * kTile, s + t0 + kTile, 4 * tma_words(t0 + kTile), &full[buf ^ 1u]);
    }
    const uint32_t nt = tma_words(t0), nall = (uint32_t)(min(e, t0 + kTile) - t0);
    mbar_wait(&full[buf], (it >> 1) & 1u);
    // thread's words: uint4 (threadIdx.x + NT * u) of the tile
    const auto word4 = [&](uint32_t u, uint32_t (&w)[4]) {
      const uint32_t i = 4 * (threadIdx.x + NT * u);
      if (i + 4 <= nt) {
        const uint4 v = *reinterpret_cast<const uint4*>(raw + i);
        w[0] = v.x; w[1] = v.y; w[2] = v.z; w[3] = v.w;
      } else {
#pragma unroll
        for (int q = 0; q < 4; q++) w[q] = i + q < nt ? raw[i + q] : (i + q < nall ? s[t0 + i + q] : 0xffffffffu);
      }
    };
    uint32_t rb[kPV];  // rb = counter << 16 | rank within the counter (invalid words: bucket B)
#pragma unroll
    for (uint32_t u = 0; u < kPV / 4; u++) {
      uint32_t w[4];
      word4(u, w);
#pragma unroll
      for (uint32_t q = 0; q < 4; q++) {
        const uint32_t ci = (w[q] < pnr ? pbucket(w[q]) : B) * kPSub + sub;  // branch-free (a predicated
        rb[4 * u + q] = (ci << 16) | atomicAdd(&th[ci], 1u);                    // atomic compiled to a branch)
      }
    }
    __syncthreads();  // A: ranks done (and the previous tile's write-out)
    uint32_t x[kPSub], v = 0;  // bucket bt's counters ([0, B]: B = the invalid words, staged last)
#pragma unroll
    for (uint32_t j = 0; j < kPSub; j++) {
      x[j] = 0;
      if (bt <= B) { x[j] = th[bt * kPSub + j]; th[bt * kPSub + j] = 0; }
      v += x[j];
    }
    uint32_t inc = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
      if (lane >= o) inc += y;
    }
    if (lane == 31) wsum[warp] = inc;
    __syncthreads();  // B
    uint32_t wpre = 0;  // exclusive prefix of this warp's total (every warp scans the NT / 32
                        // totals itself: no second barrier)
    {
      const uint32_t y = lane < NT / 32 ? wsum[lane] : 0u;
      uint32_t yi = y;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t z = __shfl_up_sync(0xffffffffu, yi, o);
        if (lane >= o) yi += z;
      }
      wpre = __shfl_sync(0xffffffffu, yi - y, warp);
    }
    uint32_t ex = wpre + inc - v;  // tile offset of bucket bt
    if (bt <= B) {
      dst[bt] = cur - (Off)ex;
      cur += (Off)v;
#pragma unroll
      for (uint32_t j = 0; j < kPSub; j++) {
        tcnt[bt * kPSub + j] = (uint16_t)ex;
        ex += x[j];
      }
    }
    __syncthreads();  // C: offsets ready
#pragma unroll
    for (uint32_t u = 0; u < kPV / 4; u++) {  // loads of a group before its stores (stage / tcnt
      uint32_t w[4], tc[4];                   // could alias for the compiler)
      word4(u, w);
#pragma unroll
      for (uint32_t q = 0; q < 4; q++) tc[q] = tcnt[rb[4 * u + q] >> 16];
#pragma unroll
      for (uint32_t q = 0; q < 4; q++) stage[tc[q] + (rb[4 * u + q] & 0xffffu)] = w[q];
    }
    __syncthreads();  // D: staged
    const uint32_t nv = tcnt[B * kPSub];  // the valid words of the tile
#pragma unroll
    for (uint32_t k0 = 0; k0 < kPV; k0 += 8) {  // eight entries per thread in flight
      uint32_t y[8];
      Off d[8];
#pragma unroll
      for (uint32_t k = 0; k < 8; k++) {
        const uint32_t p = threadIdx.x + NT * (k0 + k);
        y[k] = p < nv ? stage[p] : 0u;
      }
#pragma unroll
      for (uint32_t k = 0; k < 8; k++) d[k] = dst[pbucket(y[k])];
#pragma unroll
      for (uint32_t k = 0; k < 8; k++) {
        const uint32_t p = threadIdx.x + NT * (k0 + k);
        if (p < nv) out[(Off)(d[k] + p)] = (uint16_t)(y[k] & (kPBins - 1u));
      }
    }
  }
}

// per CTA: uint4 [c0, c1) of the partitioned array (8 entries each, never across buckets), bucket
// by bucket; bucket b's entries are offsets of bins [b << kPBits, ...) (padding kPPad is counted
// into a spare word). 32-bit counters: exact, no drains.
__global__ void __launch_bounds__(kPHT, 1)
    k_pbucket_hist(const uint16_t* __restrict__ ps, const unsigned long long* __restrict__ bstart, uint32_t B,
                   uint64_t chunk4, uint32_t pnr, Div dv, int32_t* __restrict__ H) {
  extern __shared__ uint32_t tab[];  // kPBins counters + 32 spare words
  for (uint32_t i = threadIdx.x; i < kPBins + 32; i += kPHT) tab[i] = 0;
  __syncthreads();
  const uint4* s4 = reinterpret_cast<const uint4*>(ps);
  const uint64_t end4 = bstart[B] / 8;
  const uint64_t c0 = blockIdx.x * chunk4, c1 = min(end4, c0 + chunk4);
  if (c0 >= c1) return;
  const uint32_t spare = kPBins + (threadIdx.x & 31u);
  // first bucket touching c0: last b with bstart[b] / 8 <= c0
  uint32_t lo = 0, hi = B;
  while (hi - lo > 1) {
    const uint32_t mid = (lo + hi) >> 1;
    if (bstart[mid] / 8 <= c0) lo = mid;
    else hi = mid;
  }
  const auto add8 = [&](const uint4 v) {
    const uint32_t x[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
    for (int q = 0; q < 4; q++) {
      const uint32_t o0 = x[q] & 0xffffu, o1 = x[q] >> 16;
      atomicAdd(tab + (o0 < kPBins ? o0 : spare), 1u);
      atomicAdd(tab + (o1 < kPBins ? o1 : spare), 1u);
    }
  };
  for (uint32_t b = lo; b < B; b++) {
    const unsigned long long bs = bstart[b];
    if (bs / 8 >= c1) break;
    const uint64_t a4 = max(c0, (uint64_t)(bs / 8)), e4 = min(c1, (uint64_t)(bstart[b + 1] / 8));
    if (a4 >= e4) continue;
    uint64_t i = a4 + threadIdx.x;
    constexpr int kU = 4;  // 128-bit loads in flight per thread
    for (; i + (kU - 1) * kPHT < e4; i += kU * kPHT) {
      uint4 v[kU];
#pragma unroll
      for (int u = 0; u < kU; u++) v[u] = ld_stream(s4 + i + u * kPHT);
#pragma unroll
      for (int u = 0; u < kU; u++) add8(v[u]);
    }
    for (; i < e4; i += kPHT) add8(__ldg(s4 + i));
    __syncthreads();
    // flush bucket b into H and zero the table (the bins of bucket b are counted only by the CTAs
    // whose range overlaps its region: L2 reductions)
    const uint32_t base = b << kPBits, lim = min(kPBins, pnr - base);
    if (dv.row == dv.d && (reinterpret_cast<uintptr_t>(H) & 7u) == 0) {  // compact rows: bin pairs
      unsigned long long* H2 = reinterpret_cast<unsigned long long*>(H + base);  // base is even
      uint2* t2 = reinterpret_cast<uint2*>(tab);
      for (uint32_t i2 = threadIdx.x; 2 * i2 < lim; i2 += kPHT) {
        const uint2 t = t2[i2];
        if (t.x | t.y) {
          t2[i2] = make_uint2(0u, 0u);
          if (2 * i2 + 1 < lim) atomicAdd(H2 + i2, (unsigned long long)t.x | ((unsigned long long)t.y << 32));
          else atomicAdd(H + base + 2 * i2, (int32_t)t.x);
        }
      }
    } else {
      for (uint32_t j = threadIdx.x; j < lim; j += kPHT) {
        const uint32_t t = tab[j];
        if (t) {
          tab[j] = 0;
          atomicAdd(H + hidx(base + j, dv), (int32_t)t);
        }
      }
    }
    __syncthreads();
  }
}

}  // namespace

gs_status pack_samples_run(gs_ctx* c, const uint32_t* d_raw, uint64_t n, uint32_t* d_words,
                           unsigned long long* d_n_invalid) {
  if (!n) return GS_OK;
  const uint64_t want = (n + 4 * 256 - 1) / (4 * 256);   // a thread per 4 records, at most 32 CTAs per SM
  int dev_sms = 148;
  cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, c->device);
  const unsigned grid = (unsigned)std::max<uint64_t>(1, std::min<uint64_t>(want, (uint64_t)dev_sms * 8));
  k_pack<<<grid, 256, 0, c->stream>>>(d_raw, n, c->d_kd, c->n_kernels, c->cfg.n_reasons, d_words, d_n_invalid);
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

gs_status counts_run(gs_ctx* c, const uint32_t* d_recs, uint64_t n, int32_t* d_hist, unsigned long long* d_n_invalid,
                     int accumulate) {
  cudaStream_t st = c->stream;
  const uint32_t row = c->cfg.hist_row;
  if (!accumulate && c->n_instr) GS_CUDA(c, cudaMemsetAsync(d_hist, 0, c->n_instr * row * 4, st));
  if (!n) return GS_OK;
  if (reinterpret_cast<uintptr_t>(d_recs) & 15u) return fail(c, GS_E_INVAL, "count records must be 16-byte aligned");
  int dev_sms = 148;
  cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, c->device);
  const uint64_t blocks = std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)dev_sms * 8, (n + 255) / 256));
  k_counts<<<(unsigned)blocks, 256, 0, st>>>(reinterpret_cast<const uint4*>(d_recs), n, c->d_kd, c->n_kernels,
                                             c->cfg.n_reasons, row, d_hist, d_n_invalid);
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

gs_status counts8_run(gs_ctx* c, const void* d_recs, uint64_t n, int32_t* d_hist, unsigned long long* d_n_invalid,
                      int accumulate) {
  cudaStream_t st = c->stream;
  const uint32_t row = c->cfg.hist_row, nr = c->cfg.n_reasons;
  if (!accumulate && c->n_instr) GS_CUDA(c, cudaMemsetAsync(d_hist, 0, c->n_instr * row * 4, st));
  if (!n) return GS_OK;
  int dev_sms = 148;
  cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, c->device);
  const uint64_t blocks = std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)dev_sms * 8, (n + 255) / 256));
  k_counts8<<<(unsigned)blocks, 256, 0, st>>>(static_cast<const uint2*>(d_recs), n, (uint32_t)c->n_instr * nr,
                                              make_div(nr, row), d_hist, d_n_invalid);
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

// GS_HIST_PARTITION (see the kernels): partition by bucket, then count each bucket in its table.
// d_words is 16-byte aligned here (hist_run peeled the head); the histogram is already zeroed.
gs_status partition_run(gs_ctx* c, const uint32_t* d_words, uint64_t n, int32_t* d_hist,
                        unsigned long long* d_n_invalid, int dev_sms) {
  cudaStream_t st = c->stream;
  const uint32_t P = (uint32_t)c->n_instr, nr = c->cfg.n_reasons;
  const Div dv = make_div(nr, c->cfg.hist_row);
  const uint64_t pnr = (uint64_t)P * nr;
  const uint32_t B = (uint32_t)((pnr + kPBins - 1) >> kPBits);
  if (B >= kPMaxBuckets) return GS_E_RANGE;  // caller falls back to WINDOW (2^25 bins or more)
  const uint64_t nchunk = std::max<uint64_t>(
      1, std::min<uint64_t>((uint64_t)dev_sms, (n + kSTile - 1) / kSTile));
  uint64_t chunk = (n + nchunk - 1) / nchunk;
  chunk = (chunk + kSTile - 1) / kSTile * kSTile;  // whole scatter tiles (a multiple of 4 words)
  const uint64_t nch = (n + chunk - 1) / chunk;
  // scratch: counts/offsets [nch][B] u32, bucket starts [B + 1] u64, partitioned 16-bit copy
  // (+ padding to whole uint4 per bucket)
  const uint64_t need = nch * B * 4 + 256 + (B + 1) * 8 + 256 + (n + 8ull * B + 8) * 2;
  if (c->part_bytes < need) {
    if (c->d_part) cudaFree(c->d_part);
    c->d_part = nullptr;
    c->part_bytes = 0;
    GS_CUDA(c, cudaMalloc(&c->d_part, need));
    c->part_bytes = need;
  }
  char* p = static_cast<char*>(c->d_part);
  uint32_t* cnt = reinterpret_cast<uint32_t*>(p);
  p += (nch * B * 4 + 255) / 256 * 256;
  unsigned long long* bstart = reinterpret_cast<unsigned long long*>(p);
  p += ((B + 1) * 8 + 255) / 256 * 256;
  uint16_t* ps = reinterpret_cast<uint16_t*>(p);
  k_pcount<<<(unsigned)nch, kPT, 0, st>>>(d_words, n, chunk, (uint32_t)pnr, B, cnt, d_n_invalid);
  count_launch();
  k_pscan<<<1, kPT, 0, st>>>(cnt, (uint32_t)nch, B, bstart, ps);
  count_launch();
  // 32-bit destination bases when the copy has < 2^32 entries (GS_PART_WIDE=1 forces the 64-bit
  // kernel: tests)
  const bool wide = n + 8ull * B + 8 >= (1ull << 32) || getenv("GS_PART_WIDE") != nullptr;
  const auto kern = wide ? k_pscatter<kPST, unsigned long long> : k_pscatter<kPST, uint32_t>;
  GS_CUDA(c, cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)(3 * kSTile * 4)));
  kern<<<(unsigned)nch, kPST, 3 * kSTile * 4, st>>>(d_words, n, chunk, (uint32_t)pnr, B, cnt, bstart, ps);
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  const uint64_t total4 = (n + 8ull * B + 7) / 8;  // upper bound of the padded array in uint4
  const uint64_t chunk4 = (total4 + dev_sms - 1) / dev_sms;
  const size_t smem = (size_t)(kPBins + 32) * 4;
  GS_CUDA(c, cudaFuncSetAttribute(k_pbucket_hist, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
  k_pbucket_hist<<<(unsigned)dev_sms, kPHT, smem, st>>>(ps, bstart, B, chunk4, (uint32_t)pnr, dv, d_hist);
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  c->last_hist_mode = GS_HIST_PARTITION;
  c->last_hist_bits = 32;
  c->last_hist_table_words = kPBins;
  return GS_OK;
}

gs_status hist_run(gs_ctx* c, const uint32_t* d_words, uint64_t n, int32_t* d_hist, unsigned long long* d_n_invalid,
                   int accumulate, bool zero_first) {
  cudaStream_t st = c->stream;
  const uint32_t P = (uint32_t)c->n_instr, nr = c->cfg.n_reasons;
  const Div dv = make_div(nr, c->cfg.hist_row);
  const uint64_t hbins = (uint64_t)P * c->cfg.hist_row;
  if (reinterpret_cast<uintptr_t>(d_words) & 3u) return fail(c, GS_E_INVAL, "sample pointer must be 4-byte aligned");
  if (!c->dev_sms) GS_CUDA(c, cudaDeviceGetAttribute(&c->dev_sms, cudaDevAttrMultiProcessorCount, c->device));
  const int dev_sms = c->dev_sms;
  // the pass's GPU time (gs_last_attribute_ms): from here to the end of its enqueued work
  if (!c->ev_pass[0]) {
    GS_CUDA(c, cudaEventCreate(&c->ev_pass[0]));
    GS_CUDA(c, cudaEventCreate(&c->ev_pass[1]));
  }
  c->pass_timed = false;
  GS_CUDA(c, cudaEventRecord(c->ev_pass[0], st));
  // peel the words before the first 16-byte boundary so the main kernels use 128-bit loads
  const uint64_t head = std::min<uint64_t>(n, ((16u - (reinterpret_cast<uintptr_t>(d_words) & 15u)) & 15u) / 4u);
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
  // the histogram's zeroing: folded into k_plan for the WINDOW strategy (one launch instead of a
  // memset node + k_plan), else a memset; the head words go in after it
  const bool zero = zero_first && !accumulate && hbins;
  const bool fold_zero = zero && n > head && mode == GS_HIST_WINDOW && (reinterpret_cast<uintptr_t>(d_hist) & 15u) == 0 &&
                         (n - head) / (2ull * kMinTableWords) + 1 > 1;
  if (zero && !fold_zero) GS_CUDA(c, cudaMemsetAsync(d_hist, 0, hbins * 4, st));
  const uint32_t* const d_head = d_words;
  const auto peel = [&, d_head]() -> gs_status {
    if (head) {
      k_hist_global<<<1, 32, 0, st>>>(d_head, head, P * nr, dv, d_hist, d_n_invalid);
      count_launch();
      GS_CUDA(c, cudaGetLastError());
    }
    return GS_OK;
  };
  if (!fold_zero) {
    const gs_status ps = peel();
    if (ps != GS_OK) return ps;
  }
  d_words += head;
  n -= head;
  if (!n) return GS_OK;
  const uint32_t n_ranges = ranges(bits == 16 ? nslots16 : nslots32);
  if (mode == GS_HIST_PRIVATE && n_ranges > 64) mode = GS_HIST_WINDOW;
  c->last_hist_mode = (int)mode;
  c->last_hist_bits = mode == GS_HIST_GLOBAL ? 0 : (int)bits;
  if (mode == GS_HIST_GLOBAL) {
    const uint64_t blocks = std::max<uint64_t>(
        1, std::min<uint64_t>((uint64_t)dev_sms * 4, (n + kThreadsGlobal * 4 - 1) / (kThreadsGlobal * 4)));
    k_hist_global<<<(unsigned)blocks, kThreadsGlobal, 0, st>>>(d_words, n, P * nr, dv, d_hist, d_n_invalid);
    count_launch();
    GS_CUDA(c, cudaGetLastError());
    return GS_OK;
  }
  if (mode == GS_HIST_PARTITION) {
    const gs_status ps = partition_run(c, d_words, n, d_hist, d_n_invalid, dev_sms);
    if (ps != GS_E_RANGE) return ps;
    mode = GS_HIST_WINDOW;  // more than 2048 bucket tables: the windowed strategy instead
    bits = max_kn > nslots32 ? 16 : 32;
    c->last_hist_mode = (int)mode;
    c->last_hist_bits = (int)bits;
  }
  const bool dyn = mode == GS_HIST_WINDOW;
  // WINDOW: a table just large enough for the largest kernel (+1 slot for the even window base).
  // The rest of the SM's 256 KB stays L1, which stages the counters' in-flight 128-bit loads: with
  // a 224-KB table the L1 (~28 KB) capped the loads in flight and the pass ran 30% slower.
  uint32_t tw = kTableWords;
  if (dyn) {
    const uint64_t need = bits == 16 ? ((uint64_t)(max_kn + 1) * nr + 1) / 2 : (uint64_t)(max_kn + 1) * nr;
    tw = (uint32_t)std::min<uint64_t>(kTableWords, (std::max<uint64_t>(need, kMinTableWords) + 31) & ~31ull);
  }
  c->last_hist_table_words = tw;
  const size_t smem = (size_t)(tw + 32) * 4;
  uint64_t chunks;
  if (dyn) {
    chunks = std::max<uint64_t>(1, std::min<uint64_t>((uint64_t)dev_sms, n / (2ull * tw) + 1));
  } else {
    chunks = std::max<uint64_t>(1, (uint64_t)dev_sms / n_ranges);
    chunks = std::min<uint64_t>(chunks, std::max<uint64_t>(1, n / (2ull * kTableWords)));
  }
  uint64_t chunk = (n + chunks - 1) / chunks;
  chunk = (chunk + 3) & ~3ull;
  chunks = (n + chunk - 1) / chunk;
  if (dyn) {  // work-stealing tile queue (one 64-bit word per chunk) + chunk bounds (k_plan); two
              // deferral ring halves per CTA
    GS_CUDA(c, dev_grow(&c->d_tileq, &c->tileq_cap, 2 * chunks + 1));
    GS_CUDA(c, dev_grow(&c->d_defer, &c->defer_cap, chunks * 2 * kDeferCap));
    const uint32_t nslots = (uint32_t)std::max<uint64_t>(1, (bits == 16 ? 2ull * tw : (uint64_t)tw) / nr);
    k_plan<<<fold_zero ? (uint32_t)dev_sms : 1u, 1024, 0, st>>>(d_words, n, P * nr, dv, nslots, (uint32_t)chunks,
                                                               c->d_tileq, fold_zero ? d_hist : nullptr, hbins);
    count_launch();
    if (fold_zero) {
      const gs_status ps = peel();
      if (ps != GS_OK) return ps;
    }
  }
  const auto prep = [&](auto kern) -> gs_status {  // the dynamic smem limit, raised once per kernel and size
    const void* fn = reinterpret_cast<const void*>(kern);
    int slot = -1;
    for (int q = 0; q < 4 && slot < 0; q++)
      if (c->smem_fn[q] == fn || !c->smem_fn[q]) slot = q;
    if (slot >= 0 && c->smem_fn[slot] == fn && c->smem_set[slot] >= smem) return GS_OK;
    GS_CUDA(c, cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem));
    if (slot >= 0) {
      c->smem_fn[slot] = fn;
      c->smem_set[slot] = smem;
    }
    return GS_OK;
  };
  gs_status ls = GS_OK;
  if (dyn) {
    const auto kern = bits == 16 ? k_hist_window<true> : k_hist_window<false>;
    ls = prep(kern);
    if (ls == GS_OK)
      kern<<<(uint32_t)chunks, kThreads, smem, st>>>(d_words, n, P, nr, dv, c->d_kd, c->n_kernels, 1u, d_hist,
                                                     d_n_invalid, c->d_tileq, c->d_defer, tw);
  } else {
    const auto kern = bits == 16 ? k_hist_smem<true> : k_hist_smem<false>;
    ls = prep(kern);
    if (ls == GS_OK)
      kern<<<(uint32_t)(chunks * n_ranges), kThreads, smem, st>>>(d_words, n, P, nr, dv, n_ranges, chunk, 1u, d_hist,
                                                                  d_n_invalid);
  }
  if (ls != GS_OK) return ls;
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

void attrib_free(gs_ctx* c) {
  if (c->d_part) cudaFree(c->d_part);
  c->d_part = nullptr;
  c->part_bytes = 0;
  if (c->d_tileq) cudaFree(c->d_tileq);
  c->d_tileq = nullptr;
  c->tileq_cap = 0;
  if (c->d_defer) cudaFree(c->d_defer);
  c->d_defer = nullptr;
  c->defer_cap = 0;
  for (int b = 0; b < 2; b++) {
    if (c->h_stage[b]) cudaFreeHost(c->h_stage[b]);
    if (c->d_stage[b]) cudaFree(c->d_stage[b]);
    if (c->ev_stage[b]) cudaEventDestroy(c->ev_stage[b]);
    if (c->ev_pass[b]) cudaEventDestroy(c->ev_pass[b]);
    c->ev_pass[b] = nullptr;
    if (c->ev_copied[b]) cudaEventDestroy(c->ev_copied[b]);
    c->h_stage[b] = nullptr;
    c->d_stage[b] = nullptr;
    c->ev_stage[b] = nullptr;
    c->ev_copied[b] = nullptr;
  }
  if (c->copy_stream) cudaStreamDestroy(c->copy_stream);
  c->copy_stream = nullptr;
  c->stage_words = 0;
}

}  // namespace gs
