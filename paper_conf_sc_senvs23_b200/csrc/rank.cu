// rank.cu — join of the histogram onto the flagged sites and their ranking
// (§3.2; rank key R20).
//
//   k_ktot   per detected kernel: total samples of the kernel (denominator of tot/ktot), 128-bit
//            loads, several CTAs per kernel.
//   The histogram may be a slice (rows of slots [slot0, ...)) of width 32 or R (gs_config.hist_row).
//   k_join   per site: tot = sum of the site PC's row, rel = sum over REL(rule) (P:556-563,
//            P:616-624; CONV: all reasons); running maxima of rel and tot.
//   sort     the sites enter in (kernel, idx, rule) order, so a STABLE ascending sort on
//            (maxR - rel, maxT - tot) yields the total order (rel desc, tot desc, kernel, idx,
//            rule). When bits(maxR) + bits(maxT) <= 64 the two fields are packed into one 64-bit
//            key and sorted once over exactly those bits (CUB onesweep radix sort); otherwise two
//            stable passes (by tot, then by rel).
//   k_emit   the first k rows as gs_ranked_site (one warp per row).
#include <cooperative_groups.h>
#include <cub/device/device_radix_sort.cuh>
#include <cuda_runtime.h>

#include <algorithm>

#include "ctx.h"

namespace gs {
namespace {

__constant__ uint32_t kRelMask[7] = {
    1u << 6,                // VEC   long_scoreboard
    (1u << 6) | (1u << 5),  // SPILL long_scoreboard + lg_throttle
    1u << 6,                // SHMEM long_scoreboard (R: pre-change global-load latency)
    1u << 5,                // GATOM lg_throttle
    1u << 6,                // RO    long_scoreboard (reading)
    (1u << 6) | (1u << 16), // TEX   long_scoreboard + tex_throttle
    0xffffffffu,            // CONV  all reasons (reading)
};

constexpr int kKtotThreads = 512;
constexpr uint32_t kKtotSlotsPerCta = 1024;  // 128 KB of histogram per CTA

// grid.x = kernel - kb, grid.y = slice of the kernel's slots. H holds rows of width `row` from slot
// slot0 on; a kernel's rows are one contiguous int32 range, read with 128-bit loads between a
// scalar head and tail (compact rows of R < 32 bins are not 16-byte aligned per slot).
__global__ void __launch_bounds__(kKtotThreads) k_ktot(const int32_t* __restrict__ H, uint32_t slot0, uint32_t row,
                                                       const KDesc* __restrict__ kd, uint32_t kb, uint32_t ke,
                                                       unsigned long long* __restrict__ ktot) {
  const uint32_t k = kb + blockIdx.x;
  if (k >= ke) return;
  const KDesc K = kd[k];
  const uint32_t s0 = blockIdx.y * kKtotSlotsPerCta;
  if (s0 >= K.n) return;
  const uint32_t s1 = min(K.n, s0 + kKtotSlotsPerCta);
  const uint64_t e0 = (uint64_t)(K.first - slot0 + s0) * row, e1 = (uint64_t)(K.first - slot0 + s1) * row;
  const uint64_t mis = (uint64_t)(reinterpret_cast<uintptr_t>(H) >> 2) & 3u;  // H is 4-byte aligned
  const uint64_t up = ((e0 + mis + 3) & ~(uint64_t)3) - mis, dn = ((e1 + mis) & ~(uint64_t)3) - mis;
  const uint64_t a0 = up < e1 ? up : e1;
  const uint64_t a1 = dn > a0 ? dn : a0;
  unsigned long long s = 0;
  for (uint64_t i = e0 + threadIdx.x; i < a0; i += blockDim.x) s += (uint32_t)__ldg(H + i);
  for (uint64_t i = a1 + threadIdx.x; i < e1; i += blockDim.x) s += (uint32_t)__ldg(H + i);
  const int4* h4 = reinterpret_cast<const int4*>(H + a0);
  const uint64_t n4 = (a1 - a0) / 4;
  for (uint64_t i = threadIdx.x; i < n4; i += blockDim.x) {
    const int4 v = __ldg(h4 + i);
    s += (uint32_t)v.x + (uint64_t)(uint32_t)v.y + (uint32_t)v.z + (uint64_t)(uint32_t)v.w;
  }
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  __shared__ unsigned long long ws[kKtotThreads / 32];
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
    for (int w = 0; w < kKtotThreads / 32; w++) t += ws[w];
    atomicAdd(ktot + k, t);
  }
}

// PC join (R18): one warp per 4 sites (8 lanes per site, 4 reasons per lane), rows read
// coalesced; running maxima of rel and tot for the packed sort key.
__global__ void __launch_bounds__(256) k_join(const gs_site* __restrict__ sites, uint64_t ns, const int32_t* __restrict__ H, uint32_t slot0,
                       uint32_t row, const KDesc* __restrict__ kd, unsigned long long* __restrict__ rel_out,
                       unsigned long long* __restrict__ tot_out, unsigned long long* __restrict__ mx) {
  const uint32_t lane = threadIdx.x & 31u, sub = lane & 7u;
  const uint64_t s = (blockIdx.x * (uint64_t)blockDim.x + threadIdx.x) >> 3;
  unsigned long long tot = 0, rel = 0;
  if (s < ns) {
    const gs_site st = sites[s];
    const uint64_t slot = (uint64_t)__ldg(&kd[st.kernel].first) + st.idx - slot0;
    const uint32_t m = kRelMask[st.rule];
    const int32_t* r1 = H + slot * row;
#pragma unroll
    for (uint32_t t = sub; t < 32; t += 8) {
      if (t < row) {
        const uint32_t c = (uint32_t)__ldg(r1 + t);
        tot += c;
        if ((m >> t) & 1u) rel += c;
      }
    }
  }
#pragma unroll
  for (int o = 4; o; o >>= 1) {  // within the 8 lanes of a site
    tot += __shfl_xor_sync(0xffffffffu, tot, o);
    rel += __shfl_xor_sync(0xffffffffu, rel, o);
  }
  if (s < ns && sub == 0) {
    rel_out[s] = rel;
    tot_out[s] = tot;
  }
  unsigned long long mr = rel, mt = tot;
  for (int o = 16; o >= 8; o >>= 1) {
    mr = max(mr, __shfl_xor_sync(0xffffffffu, mr, o));
    mt = max(mt, __shfl_xor_sync(0xffffffffu, mt, o));
  }
  // one pair of atomics per CTA: the maxima go to two addresses every CTA updates
  __shared__ unsigned long long bm[2][8];
  const uint32_t w = threadIdx.x >> 5;
  if (lane == 0) { bm[0][w] = mr; bm[1][w] = mt; }
  __syncthreads();
  if (threadIdx.x == 0) {
    for (uint32_t v = 1; v < (blockDim.x >> 5); v++) { mr = max(mr, bm[0][v]); mt = max(mt, bm[1][v]); }
    atomicMax(mx, mr);
    atomicMax(mx + 1, mt);
  }
}

// GS_JOIN_LINE (R33): one warp per site, lane = reason; the site's row is the sum of
// the rows of its source-line group (CSR goff/gslot), or its own PC row without line info.
// GS_JOIN_CONSUMER (R37): lgrp == nullptr, the group of a slot is the slot itself (its own row
// and its consumers' rows).
__global__ void k_join_line(const gs_site* __restrict__ sites, uint64_t ns, const int32_t* __restrict__ H,
                            uint32_t slot0, uint32_t row, const KDesc* __restrict__ kd,
                            const uint32_t* __restrict__ lgrp, const uint32_t* __restrict__ goff,
                            const uint32_t* __restrict__ gslot, unsigned long long* __restrict__ rel_out,
                            unsigned long long* __restrict__ tot_out, uint32_t* __restrict__ jrow,
                            unsigned long long* __restrict__ mx) {
  const uint64_t s = blockIdx.x * (uint64_t)(blockDim.x >> 5) + (threadIdx.x >> 5);
  if (s >= ns) return;
  const uint32_t lane = threadIdx.x & 31u;
  const gs_site st = sites[s];
  const uint32_t slot = kd[st.kernel].first + st.idx;
  const uint32_t g = lgrp ? lgrp[slot] : slot;
  unsigned long long v = 0;
  if (g == ~0u) {
    if (lane < row) v = (uint32_t)__ldg(H + (uint64_t)(slot - slot0) * row + lane);
  } else {
    for (uint32_t q = goff[g]; q < goff[g + 1]; q++)
      if (lane < row) v += (uint32_t)__ldg(H + (uint64_t)(__ldg(gslot + q) - slot0) * row + lane);
  }
  const uint32_t m = kRelMask[st.rule];
  unsigned long long tot = v, rel = ((m >> lane) & 1u) ? v : 0;
  for (int o = 16; o; o >>= 1) {
    tot += __shfl_xor_sync(0xffffffffu, tot, o);
    rel += __shfl_xor_sync(0xffffffffu, rel, o);
  }
  jrow[s * 32 + lane] = v > 0xffffffffull ? 0xffffffffu : (uint32_t)v;
  if (lane == 0) {
    rel_out[s] = rel;
    tot_out[s] = tot;
    atomicMax(mx, rel);
    atomicMax(mx + 1, tot);
  }
}

// key = ((maskR - rel) << bt) | (maskT - tot); vals = site index
__global__ void k_keys_packed(const unsigned long long* __restrict__ rel, const unsigned long long* __restrict__ tot,
                              uint64_t ns, int bt, unsigned long long mask_r, unsigned long long mask_t,
                              unsigned long long* __restrict__ keys, uint32_t* __restrict__ vals) {
  const uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (s >= ns) return;
  keys[s] = ((mask_r - rel[s]) << bt) | (mask_t - tot[s]);
  vals[s] = (uint32_t)s;
}

// ---------------------------------------------------------------- cluster sort (small site sets)
// For up to kCsMax sites whose packed key leaves kCsIdxBits free bits, the whole sort runs in ONE
// launch of a 16-CTA thread-block cluster: element = (key << 17) | site index, 8192 per CTA in
// shared memory; per 6-bit digit (LSD, stable): warp-level ranks by __match_any_sync over rows of
// 32 elements in order, per-digit prefixes over the warps, the cluster's digit totals read through
// distributed shared memory, and every element stored straight into its destination CTA's other
// buffer (st.shared::cluster); one cluster barrier per pass. The CUB onesweep path launched a
// histogram, a scan and one kernel per 8-bit digit over global memory.
namespace cg = cooperative_groups;
constexpr uint32_t kCsCtas = 16, kCsThreads = 1024, kCsWarps = kCsThreads / 32, kCsRows = 8;
constexpr uint32_t kCsPer = kCsWarps * kCsRows * 32;     // elements per CTA (8192)
constexpr uint32_t kCsMax = kCsCtas * kCsPer;            // 131072 sites
constexpr uint32_t kCsIdxBits = 17;                      // site index bits (kCsMax = 2^17)
#ifndef GS_CS_DIGIT_BITS
#define GS_CS_DIGIT_BITS 6
#endif
constexpr uint32_t kCsDigitBits = GS_CS_DIGIT_BITS, kCsDigits = 1u << kCsDigitBits;
constexpr uint32_t kCsDpl = kCsDigits / 32;  // digits per lane in the base scan
static_assert(kCsDigits >= 32 && kCsDigits <= 256, "digit width");
static_assert(kCsMax == (1u << kCsIdxBits), "index field");

__global__ void __launch_bounds__(kCsThreads, 1)
    k_cluster_sort(  // launched as one cluster of kCsCtas CTAs
const unsigned long long* __restrict__ rel, const unsigned long long* __restrict__ tot, uint32_t ns,
                   int bt, unsigned long long mask_r, unsigned long long mask_t, uint32_t bits,
                   uint32_t* __restrict__ order) {
  extern __shared__ unsigned long long cs_buf[];          // [2][kCsPer]
  __shared__ uint32_t wc[kCsWarps][kCsDigits];            // per-warp digit counts -> exclusive prefixes
  __shared__ uint32_t cnt[kCsDigits];                     // this CTA's digit totals (read by the cluster)
  __shared__ uint32_t allc[kCsCtas][kCsDigits];
  __shared__ uint32_t base[kCsDigits];
  cg::cluster_group cluster = cg::this_cluster();
  const uint32_t r = cluster.block_rank(), lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  const uint32_t lt = (1u << lane) - 1u;
  unsigned long long* cur = cs_buf;
  unsigned long long* nxt = cs_buf + kCsPer;
  // element i of CTA r is site r * kCsPer + i; warp w owns [w * 256, w * 256 + 256), row k its
  // elements w * 256 + 32 k + lane
  static_assert(kCsPer % kCsThreads == 0, "whole rows per thread");
#pragma unroll  // all of a thread's loads in flight at once
  for (uint32_t i = threadIdx.x; i < kCsPer; i += kCsThreads) {
    const uint32_t sidx = r * kCsPer + i;
    cur[i] = sidx < ns ? ((((mask_r - rel[sidx]) << bt) | (mask_t - tot[sidx])) << kCsIdxBits) | sidx : ~0ull;
  }
  __syncthreads();
  const uint32_t passes = (bits + kCsDigitBits - 1) / kCsDigitBits;
  for (uint32_t pass = 0; pass < passes; pass++) {
    const uint32_t sh = kCsIdxBits + pass * kCsDigitBits;
    for (uint32_t d = lane; d < kCsDigits; d += 32) wc[warp][d] = 0;
    __syncwarp();
    unsigned long long e[kCsRows];
    uint32_t dr[kCsRows];  // digit << 16 | rank within the warp's elements of that digit
#pragma unroll
    for (uint32_t k = 0; k < kCsRows; k++) {
      e[k] = cur[warp * kCsRows * 32 + 32 * k + lane];
      const uint32_t d = (uint32_t)(e[k] >> sh) & (kCsDigits - 1u);
      const uint32_t m = __match_any_sync(0xffffffffu, d);
      const uint32_t lead = 31u - __clz(m);  // the row's last lane of this digit adds the count
      const uint32_t before = wc[warp][d];
      __syncwarp();
      if (lane == lead) wc[warp][d] = before + __popc(m);
      __syncwarp();
      dr[k] = (d << 16) | (before + __popc(m & lt));
    }
    __syncthreads();
    for (uint32_t d = threadIdx.x; d < kCsDigits; d += kCsThreads) {  // prefixes over the warps, CTA totals
      uint32_t acc = 0;
      for (uint32_t w = 0; w < kCsWarps; w++) {
        const uint32_t x = wc[w][d];
        wc[w][d] = acc;
        acc += x;
      }
      cnt[d] = acc;
    }
    cluster.sync();  // every CTA's cnt[] is final (and every CTA finished reading its buffer)
    for (uint32_t i = threadIdx.x; i < kCsCtas * kCsDigits; i += kCsThreads) {
      const uint32_t c = i / kCsDigits, d = i % kCsDigits;
      allc[c][d] = *cluster.map_shared_rank(&cnt[d], c);
    }
    __syncthreads();
    if (threadIdx.x < 32) {  // base[d] = elements of smaller digits anywhere + of digit d in CTAs < r
      uint32_t totd[kCsDpl], mine[kCsDpl], sum = 0;
#pragma unroll
      for (uint32_t h = 0; h < kCsDpl; h++) {
        const uint32_t d = lane * kCsDpl + h;
        uint32_t t = 0, m = 0;
        for (uint32_t c = 0; c < kCsCtas; c++) {
          t += allc[c][d];
          m += c < r ? allc[c][d] : 0u;
        }
        totd[h] = t;
        mine[h] = m;
        sum += t;
      }
      uint32_t inc = sum;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= (uint32_t)o) inc += y;
      }
      uint32_t ex = inc - sum;
#pragma unroll
      for (uint32_t h = 0; h < kCsDpl; h++) {
        base[lane * kCsDpl + h] = ex + mine[h];
        ex += totd[h];
      }
    }
    __syncthreads();
#pragma unroll
    for (uint32_t k = 0; k < kCsRows; k++) {  // straight into the destination CTA's other buffer
      const uint32_t d = dr[k] >> 16;
      const uint32_t pos = base[d] + wc[warp][d] + (dr[k] & 0xffffu);
      unsigned long long* dst = cluster.map_shared_rank(nxt, pos / kCsPer);
      dst[pos % kCsPer] = e[k];
    }
    cluster.sync();  // all elements arrived; allc/cnt/wc free for the next pass
    unsigned long long* t = cur;
    cur = nxt;
    nxt = t;
  }
#pragma unroll
  for (uint32_t i = threadIdx.x; i < kCsPer; i += kCsThreads) {
    const uint32_t q = r * kCsPer + i;
    if (q < ns) order[q] = (uint32_t)(cur[i] & (kCsMax - 1u));
  }
}

// one field: key = mask - val[order[i]] (order == nullptr: identity, vals = i)
__global__ void k_keys_field(const unsigned long long* __restrict__ val, const uint32_t* __restrict__ order,
                             uint64_t ns, unsigned long long mask, unsigned long long* __restrict__ keys,
                             uint32_t* __restrict__ vals) {
  const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (i >= ns) return;
  const uint32_t s = order ? order[i] : (uint32_t)i;
  keys[i] = mask - val[s];
  if (!order) vals[i] = s;
}

// ranked rows, one thread per row (the order -> site -> kernel -> histogram-row chain of every
// row in flight at once); counts from the PC row of H, or the joined row jrow. Each thread builds
// its 168-B row in shared memory and the CTA writes its 256 rows as one contiguous, coalesced run
// of 8-byte words (per-thread row stores touched 32 lines per warp store: 21 -> 6 us on C4).
constexpr int kEmitT = 256;
constexpr uint32_t kRowWords = sizeof(gs_ranked_site) / 8;
static_assert(sizeof(gs_ranked_site) % 8 == 0, "ranked rows are whole 8-byte words");
__global__ void __launch_bounds__(kEmitT) k_emit(const uint32_t* __restrict__ order, uint64_t kk,
                                                 const gs_site* __restrict__ sites, const int32_t* __restrict__ H,
                                                 uint32_t slot0, uint32_t row, const uint32_t* __restrict__ jrow,
                                                 const unsigned long long* __restrict__ rel_a,
                                                 const unsigned long long* __restrict__ tot_a,
                                                 const KDesc* __restrict__ kd, const unsigned long long* __restrict__ ktot,
                                                 gs_ranked_site* __restrict__ out) {
  __shared__ gs_ranked_site rows[kEmitT];
  const uint64_t q0 = blockIdx.x * (uint64_t)kEmitT, q = q0 + threadIdx.x;
  if (q < kk) {
    const uint32_t si = __ldg(order + q);
    const gs_site st = sites[si];
    gs_ranked_site* r = rows + threadIdx.x;
    uint2* c2 = reinterpret_cast<uint2*>(r->counts);  // counts[] is 8-byte aligned
    if (jrow) {
      const uint4* j4 = reinterpret_cast<const uint4*>(jrow + (uint64_t)si * 32);
#pragma unroll
      for (int t = 0; t < 8; t++) {
        const uint4 v = __ldg(j4 + t);
        c2[2 * t] = make_uint2(v.x, v.y);
        c2[2 * t + 1] = make_uint2(v.z, v.w);
      }
    } else {
      const int32_t* h = H + ((uint64_t)__ldg(&kd[st.kernel].first) + st.idx - slot0) * row;
      uint32_t c[32];
#pragma unroll
      for (uint32_t t = 0; t < 32; t++) c[t] = t < row ? (uint32_t)__ldg(h + t) : 0u;
#pragma unroll
      for (int t = 0; t < 16; t++) c2[t] = make_uint2(c[2 * t], c[2 * t + 1]);
    }
    r->kernel = st.kernel;
    r->idx = st.idx;
    r->rule = st.rule;
    r->pad = 0;
    r->rel = rel_a[si];
    r->tot = tot_a[si];
    r->ktot = ktot[st.kernel];
  }
  __syncthreads();
  const uint64_t nrow = kk - q0 < (uint64_t)kEmitT ? kk - q0 : (uint64_t)kEmitT;
  const unsigned long long* src = reinterpret_cast<const unsigned long long*>(rows);
  unsigned long long* dst = reinterpret_cast<unsigned long long*>(out + q0);
  for (uint32_t i = threadIdx.x; i < nrow * kRowWords; i += kEmitT) dst[i] = src[i];
}

cudaLaunchConfig_t cluster_cfg(cudaStream_t st) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(kCsCtas);
  cfg.blockDim = dim3(kCsThreads);
  cfg.dynamicSmemBytes = 2 * kCsPer * 8;
  cfg.stream = st;
  return cfg;
}
void cluster_attr(cudaLaunchAttribute* at) {
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = kCsCtas;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
}

int bits_of(unsigned long long v) { return v ? 64 - __builtin_clzll(v) : 0; }
unsigned long long mask_of(int b) { return b >= 64 ? ~0ull : ((1ull << b) - 1); }

}  // namespace

gs_status rank_run(gs_ctx* c, const int32_t* d_hist, uint32_t slot0, uint64_t k, gs_ranked_site* out,
                   bool out_is_host, uint64_t* n_out) {
  cudaStream_t st = c->stream;
  const uint64_t ns = c->n_sites;
  const uint64_t kk = std::min<uint64_t>(k, ns);
  const uint32_t row = c->cfg.hist_row;
  const uint64_t nkt = (uint64_t)std::max<uint32_t>(c->n_kernels, 1) + 2;
  const bool cons = c->cfg.join_mode == GS_JOIN_CONSUMER;
  if (cons && !c->cons_ready) return fail(c, GS_E_STATE, "consumer join: gs_detect ran in another join mode");
  const bool line = (c->cfg.join_mode == GS_JOIN_LINE && c->n_lgroups) || cons;
  // ---- every allocation first (the enqueue below may be captured into a CUDA graph)
  if (ns > 0x7fffffffull) return fail(c, GS_E_RANGE, "more than 2^31-1 sites (the site sort takes int counts)");
  // kernel totals + the two maxima: grown with the kernel count (a later gs_load_sass may load more)
  GS_CUDA(c, dev_grow(&c->d_ktot, &c->ktot_cap, nkt));
  unsigned long long* d_max = c->d_ktot + (nkt - 2);
  size_t cub_bytes = 0;
  if (ns) {
    if (c->rank_cap < ns) {
      for (int b = 0; b < 2; b++) {
        if (c->d_rank_keys[b]) cudaFree(c->d_rank_keys[b]);
        if (c->d_rank_vals[b]) cudaFree(c->d_rank_vals[b]);
        c->d_rank_keys[b] = nullptr;
        c->d_rank_vals[b] = nullptr;
      }
      c->rank_cap = 0;
      for (int b = 0; b < 2; b++) {
        GS_CUDA(c, cudaMalloc((void**)&c->d_rank_keys[b], ns * 8));
        GS_CUDA(c, cudaMalloc((void**)&c->d_rank_vals[b], ns * 4));
      }
      c->rank_cap = ns;
    }
    cub::DeviceRadixSort::SortPairs(nullptr, cub_bytes, c->d_rank_keys[0], c->d_rank_keys[1], c->d_rank_vals[0],
                                    c->d_rank_vals[1], (int)ns, 0, 64, st);
    const size_t arr = ((ns * 8 + 255) / 256) * 256;  // rel and tot arrays live in the temp block
    if (c->sort_tmp_bytes < cub_bytes + 2 * arr) {
      if (c->d_sort_tmp) cudaFree(c->d_sort_tmp);
      c->d_sort_tmp = nullptr;
      c->sort_tmp_bytes = 0;
      GS_CUDA(c, cudaMalloc(&c->d_sort_tmp, cub_bytes + 2 * arr));
      c->sort_tmp_bytes = cub_bytes + 2 * arr;
    }
    if (line) GS_CUDA(c, dev_grow(&c->d_jrow, &c->jrow_cap, ns * 32));
    if (kk && out_is_host) GS_CUDA(c, dev_grow(&c->d_ranked, &c->ranked_cap, kk));
  }
  GS_CUDA(c, pin_grow(c, 16));
  if (c->cluster_sort_ok < 0) {  // once per context: can a 16-CTA cluster with 128 KB each run here?
    c->cluster_sort_ok = 0;
    if (cudaFuncSetAttribute(k_cluster_sort, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) == cudaSuccess &&
        cudaFuncSetAttribute(k_cluster_sort, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * kCsPer * 8) ==
            cudaSuccess) {
      cudaLaunchConfig_t cfg = cluster_cfg(st);
      cudaLaunchAttribute at[1];
      cluster_attr(at);
      cfg.attrs = at;
      cfg.numAttrs = 1;
      int nclusters = 0;
      if (cudaOccupancyMaxActiveClusters(&nclusters, k_cluster_sort, &cfg) == cudaSuccess && nclusters > 0)
        c->cluster_sort_ok = getenv("GS_NO_CLUSTER_SORT") ? 0 : 1;
    }
    cudaGetLastError();
  }
  if (!c->side_stream) {
    GS_CUDA(c, cudaStreamCreateWithFlags(&c->side_stream, cudaStreamNonBlocking));
    GS_CUDA(c, cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
    GS_CUDA(c, cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
  }
  unsigned long long* mx = static_cast<unsigned long long*>(c->h_pin);
  unsigned long long* k0 = c->d_rank_keys[0];
  unsigned long long* k1 = c->d_rank_keys[1];
  uint32_t* v0 = c->d_rank_vals[0];
  uint32_t* v1 = c->d_rank_vals[1];
  const size_t arr = ((ns * 8 + 255) / 256) * 256;
  unsigned long long* d_rel = reinterpret_cast<unsigned long long*>(c->d_sort_tmp);
  unsigned long long* d_tot = reinterpret_cast<unsigned long long*>(static_cast<char*>(c->d_sort_tmp) + arr);
  void* cub_tmp = static_cast<char*>(c->d_sort_tmp) + 2 * arr;
  const unsigned grid = (unsigned)((ns + 255) / 256);
  auto passes = [](int bits) { return (uint64_t)(bits + 7) / 8 + 2; };  // onesweep digits + hist + scan
  // sort by the packed key and emit the first kk rows
  const auto sort_emit = [&](int br, int bt) -> gs_status {
    const uint32_t* order = v0;
    size_t b1 = cub_bytes;
    if (br + bt + kCsIdxBits <= 64 && ns <= kCsMax && br + bt > 0 && c->cluster_sort_ok) {
      cudaLaunchConfig_t cfg = cluster_cfg(st);
      cudaLaunchAttribute at[1];
      cluster_attr(at);
      cfg.attrs = at;
      cfg.numAttrs = 1;
      GS_CUDA(c, cudaLaunchKernelEx(&cfg, k_cluster_sort, (const unsigned long long*)d_rel,
                                    (const unsigned long long*)d_tot, (uint32_t)ns, bt, mask_of(br), mask_of(bt),
                                    (uint32_t)(br + bt), v0));
      count_launch();
      order = v0;
    } else if (br + bt <= 64) {
      k_keys_packed<<<grid, 256, 0, st>>>(d_rel, d_tot, ns, bt, mask_of(br), mask_of(bt), k0, v0);
      count_launch();
      if (br + bt > 0) {
        cub::DoubleBuffer<unsigned long long> dk(k0, k1);
        cub::DoubleBuffer<uint32_t> dv(v0, v1);
        GS_CUDA(c, cub::DeviceRadixSort::SortPairs(cub_tmp, b1, dk, dv, (int)ns, 0, br + bt, st));
        count_launch(passes(br + bt));
        order = dv.Current();
      }
    } else {
      k_keys_field<<<grid, 256, 0, st>>>(d_tot, nullptr, ns, mask_of(bt), k0, v0);
      count_launch();
      GS_CUDA(c, cub::DeviceRadixSort::SortPairs(cub_tmp, b1, k0, k1, v0, v1, (int)ns, 0, bt, st));
      count_launch(passes(bt));
      k_keys_field<<<grid, 256, 0, st>>>(d_rel, v1, ns, mask_of(br), k0, nullptr);
      count_launch();
      b1 = cub_bytes;
      GS_CUDA(c, cub::DeviceRadixSort::SortPairs(cub_tmp, b1, k0, k1, v1, v0, (int)ns, 0, br, st));
      count_launch(passes(br));
      order = v0;
    }
    GS_CUDA(c, cudaGetLastError());
    if (kk) {
      gs_ranked_site* dst = out_is_host ? c->d_ranked : out;
      GS_CUDA(c, cudaStreamWaitEvent(st, c->ev_join, 0));  // the kernel totals (side stream)
      k_emit<<<(unsigned)((kk + kEmitT - 1) / kEmitT), kEmitT, 0, st>>>(order, kk, c->d_sites, d_hist, slot0, row,
                                                          line ? c->d_jrow : nullptr, d_rel, d_tot, c->d_kd,
                                                          c->d_ktot, dst);
      count_launch();
      GS_CUDA(c, cudaGetLastError());
      if (out_is_host)
        GS_CUDA(c, cudaMemcpyAsync(out, dst, kk * sizeof(gs_ranked_site), cudaMemcpyDeviceToHost, st));
    }
    return GS_OK;
  };
  const int gr = c->rank_bits_guess[0], gt = c->rank_bits_guess[1];
  // kernel totals, join, maxima read-back, and (with the previous call's key widths) sort + emit
  // The kernel totals (a read of the whole histogram) run on the side stream, concurrently with the
  // join and the sort; k_emit (or the end of the sequence) joins them back.
  const auto enqueue_main = [&]() -> gs_status {
    GS_CUDA(c, cudaMemsetAsync(c->d_ktot, 0, nkt * 8, st));  // (the maxima live here too)
    GS_CUDA(c, cudaEventRecord(c->ev_fork, st));
    GS_CUDA(c, cudaStreamWaitEvent(c->side_stream, c->ev_fork, 0));
    if (c->det_ke > c->det_kb) {  // kernel totals of the detected kernels only
      uint32_t max_n = 1;
      for (uint32_t q = c->det_kb; q < c->det_ke; q++) max_n = std::max(max_n, c->kd_h[q].n);
      dim3 g2(c->det_ke - c->det_kb, (max_n + kKtotSlotsPerCta - 1) / kKtotSlotsPerCta);
      k_ktot<<<g2, kKtotThreads, 0, c->side_stream>>>(d_hist, slot0, row, c->d_kd, c->det_kb, c->det_ke, c->d_ktot);
      count_launch();
      GS_CUDA(c, cudaGetLastError());
    }
    GS_CUDA(c, cudaEventRecord(c->ev_join, c->side_stream));
    if (!ns) {
      GS_CUDA(c, cudaStreamWaitEvent(st, c->ev_join, 0));
      return GS_OK;
    }
    if (line) {
      k_join_line<<<(unsigned)((ns + 7) / 8), 256, 0, st>>>(
          c->d_sites, ns, d_hist, slot0, row, c->d_kd, cons ? nullptr : c->d_lgrp, cons ? c->d_cgoff : c->d_goff,
          cons ? c->d_cgslot : c->d_gslot, d_rel, d_tot, c->d_jrow, d_max);
    } else {
      k_join<<<(unsigned)((ns * 8 + 255) / 256), 256, 0, st>>>(c->d_sites, ns, d_hist, slot0, row, c->d_kd, d_rel,
                                                               d_tot, d_max);
    }
    count_launch();
    GS_CUDA(c, cudaGetLastError());
    // The packed sort key needs the bit widths of max(rel) and max(tot). They are read back with
    // one async copy; the sort itself is enqueued right away with the widths of the previous call
    // (padded to whole radix digits, which costs no extra pass) and redone with the exact
    // widths only when this call's maxima do not fit them (one host synchronisation otherwise).
    if (gr >= 0) {
      const gs_status se = sort_emit(gr, gt);
      if (se != GS_OK) return se;
    }
    GS_CUDA(c, cudaStreamWaitEvent(st, c->ev_join, 0));  // (again after k_emit: harmless)
    // the maxima go to the host last: only the host's width check reads them (a copy between the
    // join and the sort sat on the critical path)
    GS_CUDA(c, cudaMemcpyAsync(mx, d_max, 16, cudaMemcpyDeviceToHost, st));
    return GS_OK;
  };
  // The whole sequence is replayed as one CUDA graph while its parameters repeat (e.g. one rank
  // call per step): a dozen launches of small kernels become one graph launch.
  const uintptr_t key[] = {(uintptr_t)ns, (uintptr_t)kk, (uintptr_t)d_hist, slot0, row, (uintptr_t)out,
                           out_is_host, (uintptr_t)(int64_t)gr, (uintptr_t)(int64_t)gt, line, cons, c->det_kb,
                           c->det_ke, (uintptr_t)c->d_sites, (uintptr_t)c->d_sort_tmp, (uintptr_t)k0, (uintptr_t)v0,
                           (uintptr_t)c->d_jrow, (uintptr_t)c->d_ranked, (uintptr_t)mx, (uintptr_t)c->d_ktot,
                           (uintptr_t)c->d_kd, (uintptr_t)c->d_cgoff, (uintptr_t)c->d_cgslot, (uintptr_t)c->d_goff,
                           (uintptr_t)c->d_gslot, (uintptr_t)c->d_lgrp, (uintptr_t)c->n_kernels};
  constexpr size_t nkey = sizeof(key) / sizeof(key[0]);
  static const bool no_graph = getenv("GS_NO_GRAPH") != nullptr;
  bool host_ok = true;  // a captured D2H copy needs page-locked (or device) destination memory
  if (kk && out_is_host) {
    cudaPointerAttributes pa;
    host_ok = cudaPointerGetAttributes(&pa, out) == cudaSuccess && pa.type == cudaMemoryTypeHost;
    cudaGetLastError();
  }
  // (the legacy / per-thread default streams cannot be captured: plain launches there)
  const bool capturable = st != nullptr && st != cudaStreamLegacy && st != cudaStreamPerThread;
  const bool use_graph = !no_graph && gr >= 0 && ns && host_ok && capturable;
  if (use_graph) {
    bool hit = c->rank_exec && c->rank_key.size() == nkey;
    for (size_t q = 0; hit && q < nkey; q++) hit = c->rank_key[q] == key[q];
    if (!hit) {
      if (c->rank_exec) cudaGraphExecDestroy(c->rank_exec);
      c->rank_exec = nullptr;
      const uint64_t l0 = launch_count_now();
      GS_CUDA(c, cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
      const gs_status s1 = enqueue_main();
      cudaGraph_t g = nullptr;
      const cudaError_t e = cudaStreamEndCapture(st, &g);
      if (s1 != GS_OK) {
        if (g) cudaGraphDestroy(g);
        return s1;
      }
      GS_CUDA(c, e);
      const cudaError_t ei = cudaGraphInstantiate(&c->rank_exec, g, 0);
      cudaGraphDestroy(g);
      GS_CUDA(c, ei);
      c->rank_key.assign(key, key + nkey);
      c->rank_graph_launches = launch_count_now() - l0;
      count_launch_undo(c->rank_graph_launches);  // counted again when the graph runs
    }
    GS_CUDA(c, cudaGraphLaunch(c->rank_exec, st));
    count_launch(c->rank_graph_launches);
  } else {
    const gs_status s1 = enqueue_main();
    if (s1 != GS_OK) return s1;
  }
  if (ns) {
    GS_CUDA(c, cudaStreamSynchronize(st));
    const int br = bits_of(mx[0]), bt = bits_of(mx[1]);
    if (br + bt <= 64) {  // next call's widths: this call's, slack spread to fill the last digit
      // the digit width of the sort that will run: 6-bit cluster passes or 8-bit CUB passes
      const int db = (c->cluster_sort_ok == 1 && ns <= kCsMax && br + bt + (int)kCsIdxBits <= 64) ? (int)kCsDigitBits : 8;
      const int slack = ((br + bt + db - 1) / db) * db - (br + bt);
      c->rank_bits_guess[0] = std::min(64, br + slack / 2);
      c->rank_bits_guess[1] = std::min(64, bt + slack - slack / 2);
      if (c->rank_bits_guess[0] + c->rank_bits_guess[1] > 64) c->rank_bits_guess[0] = c->rank_bits_guess[1] = -1;
    } else {
      c->rank_bits_guess[0] = c->rank_bits_guess[1] = -1;
    }
    if (gr < 0 || br > gr || bt > gt) {
      gs_status s2 = sort_emit(br, bt);
      if (s2 != GS_OK) return s2;
    }
  }
  GS_CUDA(c, cudaStreamSynchronize(st));
  if (n_out) *n_out = kk;
  return GS_OK;
}

// a new module invalidates the captured rank sequence (its k_ktot grid follows the kernel sizes)
void rank_reset_graph(gs_ctx* c) {
  if (c->rank_exec) cudaGraphExecDestroy(c->rank_exec);
  c->rank_exec = nullptr;
  c->rank_key.clear();
  c->rank_bits_guess[0] = c->rank_bits_guess[1] = -1;
}

void rank_free(gs_ctx* c) {
  if (c->rank_exec) cudaGraphExecDestroy(c->rank_exec);
  c->rank_exec = nullptr;
  c->rank_key.clear();
  for (int b = 0; b < 2; b++) {
    if (c->d_rank_keys[b]) cudaFree(c->d_rank_keys[b]);
    if (c->d_rank_vals[b]) cudaFree(c->d_rank_vals[b]);
    c->d_rank_keys[b] = nullptr;
    c->d_rank_vals[b] = nullptr;
  }
  if (c->d_sort_tmp) cudaFree(c->d_sort_tmp);
  if (c->d_ktot) cudaFree(c->d_ktot);
  if (c->d_ranked) cudaFree(c->d_ranked);
  if (c->d_jrow) cudaFree(c->d_jrow);
  c->d_jrow = nullptr;
  c->jrow_cap = 0;
  c->d_sort_tmp = nullptr;
  c->d_ktot = nullptr;
  c->ktot_cap = 0;
  c->d_ranked = nullptr;
  c->rank_cap = 0;
  c->sort_tmp_bytes = 0;
  c->ranked_cap = 0;
}

}  // namespace gs
