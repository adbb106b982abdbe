// rank.cu — join of the histogram onto the flagged sites and their ranking
// (§3.2; rank key R20).
//
//   k_ktot   per kernel: total samples of the kernel (denominator of tot/ktot).
//   k_join   per site: tot = sum of the site PC's row, rel = sum over REL(rule) (P:556-563,
//            P:616-624; CONV: all reasons). Writes ~tot / ~rel keys.
//   sort     two stable LSD radix sorts (CUB DeviceRadixSort): by ~tot, then by ~rel. The sites
//            enter in (kernel, idx, rule) order, so stability yields the total order
//            (rel desc, tot desc, kernel, idx, rule).
//   k_emit   the first k rows as gs_ranked_site.
#include <cub/device/device_radix_sort.cuh>
#include <cuda_runtime.h>

#include <algorithm>

#include "ctx.h"

namespace gs {
namespace {

// onesweep radix sort of 64-bit keys: 1 histogram + 1 exclusive-sum + 8 digit passes
constexpr uint64_t kCubSortLaunches = 10;

__constant__ uint32_t kRelMask[7] = {
    1u << 6,                // VEC   long_scoreboard
    (1u << 6) | (1u << 5),  // SPILL long_scoreboard + lg_throttle
    1u << 6,                // SHMEM long_scoreboard (R: pre-change global-load latency)
    1u << 5,                // GATOM lg_throttle
    1u << 6,                // RO    long_scoreboard (reading)
    (1u << 6) | (1u << 16), // TEX   long_scoreboard + tex_throttle
    0xffffffffu,            // CONV  all reasons (reading)
};

__global__ void k_ktot(const int32_t* __restrict__ H, const KDesc* __restrict__ kd, uint32_t nk,
                       unsigned long long* __restrict__ ktot) {
  const uint32_t k = blockIdx.x;
  if (k >= nk) return;
  const KDesc K = kd[k];
  const uint64_t a = (uint64_t)K.first * 32, e = a + (uint64_t)K.n * 32;
  unsigned long long s = 0;
  for (uint64_t i = a + threadIdx.x; i < e; i += blockDim.x) s += (uint32_t)H[i];
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  __shared__ unsigned long long ws[32];
  if ((threadIdx.x & 31) == 0) ws[threadIdx.x >> 5] = s;
  __syncthreads();
  if (threadIdx.x == 0) {
    unsigned long long t = 0;
    for (int w = 0; w < (int)(blockDim.x >> 5); w++) t += ws[w];
    ktot[k] = t;
  }
}

__global__ void k_join(const gs_site* __restrict__ sites, uint64_t ns, const int32_t* __restrict__ H,
                       const KDesc* __restrict__ kd, unsigned long long* __restrict__ key_tot,
                       unsigned long long* __restrict__ key_rel, uint32_t* __restrict__ vals) {
  const uint64_t s = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (s >= ns) return;
  const gs_site st = sites[s];
  const uint64_t slot = (uint64_t)kd[st.kernel].first + st.idx;
  const int4* row = reinterpret_cast<const int4*>(H + slot * 32);
  const uint32_t m = kRelMask[st.rule];
  unsigned long long tot = 0, rel = 0;
#pragma unroll
  for (int q = 0; q < 8; q++) {
    const int4 v = __ldg(row + q);
    const uint32_t c[4] = {(uint32_t)v.x, (uint32_t)v.y, (uint32_t)v.z, (uint32_t)v.w};
#pragma unroll
    for (int t = 0; t < 4; t++) {
      tot += c[t];
      if ((m >> (4 * q + t)) & 1u) rel += c[t];
    }
  }
  key_tot[s] = ~tot;
  key_rel[s] = ~rel;
  vals[s] = (uint32_t)s;
}

__global__ void k_gather_keys(const uint32_t* __restrict__ order, const unsigned long long* __restrict__ key_rel,
                              uint64_t ns, unsigned long long* __restrict__ out) {
  const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (i < ns) out[i] = key_rel[order[i]];
}

__global__ void k_emit(const uint32_t* __restrict__ order, uint64_t kk, const gs_site* __restrict__ sites,
                       const int32_t* __restrict__ H, const KDesc* __restrict__ kd,
                       const unsigned long long* __restrict__ ktot, gs_ranked_site* __restrict__ out) {
  const uint64_t q = blockIdx.x;  // one warp per row
  if (q >= kk) return;
  const int lane = threadIdx.x;
  const gs_site st = sites[order[q]];
  const uint64_t slot = (uint64_t)kd[st.kernel].first + st.idx;
  const uint32_t c = (uint32_t)H[slot * 32 + lane];
  const uint32_t m = kRelMask[st.rule];
  unsigned long long tot = c, rel = ((m >> lane) & 1u) ? c : 0;
  for (int o = 16; o; o >>= 1) {
    tot += __shfl_xor_sync(0xffffffffu, tot, o);
    rel += __shfl_xor_sync(0xffffffffu, rel, o);
  }
  gs_ranked_site* r = out + q;
  r->counts[lane] = c;
  if (lane == 0) {
    r->kernel = st.kernel;
    r->idx = st.idx;
    r->rule = st.rule;
    r->pad = 0;
    r->rel = rel;
    r->tot = tot;
    r->ktot = ktot[st.kernel];
  }
}

}  // namespace

gs_status rank_run(gs_ctx* c, const int32_t* d_hist, uint64_t k, gs_ranked_site* out, bool out_is_host,
                   uint64_t* n_out) {
  cudaStream_t st = c->stream;
  const uint64_t ns = c->n_sites;
  const uint64_t kk = std::min<uint64_t>(k, ns);
  if (!c->d_ktot) GS_CUDA(c, cudaMalloc((void**)&c->d_ktot, (uint64_t)std::max<uint32_t>(c->n_kernels, 1) * 8));
  if (c->n_kernels) {
    k_ktot<<<c->n_kernels, 256, 0, st>>>(d_hist, c->d_kd, c->n_kernels, c->d_ktot); count_launch();
    GS_CUDA(c, cudaGetLastError());
  }
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
      // a third key buffer holds ~rel in site order
      if (c->d_sort_tmp) cudaFree(c->d_sort_tmp);
      c->d_sort_tmp = nullptr;
      c->sort_tmp_bytes = 0;
      c->rank_cap = ns;
    }
    unsigned long long* key_tot = c->d_rank_keys[0];
    unsigned long long* key_tmp = c->d_rank_keys[1];
    uint32_t* v0 = c->d_rank_vals[0];
    uint32_t* v1 = c->d_rank_vals[1];
    // CUB temp storage also hosts the ~rel array (site order)
    size_t cub_bytes = 0;
    cub::DeviceRadixSort::SortPairs(nullptr, cub_bytes, key_tot, key_tmp, v0, v1, (int)ns, 0, 64, st);
    const size_t rel_bytes = ((ns * 8 + 255) / 256) * 256;
    if (c->sort_tmp_bytes < cub_bytes + rel_bytes) {
      if (c->d_sort_tmp) cudaFree(c->d_sort_tmp);
      c->d_sort_tmp = nullptr;
      GS_CUDA(c, cudaMalloc(&c->d_sort_tmp, cub_bytes + rel_bytes));
      c->sort_tmp_bytes = cub_bytes + rel_bytes;
    }
    unsigned long long* key_rel = reinterpret_cast<unsigned long long*>(c->d_sort_tmp);
    void* cub_tmp = static_cast<char*>(c->d_sort_tmp) + rel_bytes;
    const unsigned grid = (unsigned)((ns + 255) / 256);
    k_join<<<grid, 256, 0, st>>>(c->d_sites, ns, d_hist, c->d_kd, key_tot, key_rel, v0); count_launch();
    GS_CUDA(c, cudaGetLastError());
    size_t b1 = cub_bytes;
    GS_CUDA(c, cub::DeviceRadixSort::SortPairs(cub_tmp, b1, key_tot, key_tmp, v0, v1, (int)ns, 0, 64, st));
    count_launch(kCubSortLaunches);
    // v1 = sites ordered by tot desc (stable); now sort by rel desc, stable
    k_gather_keys<<<grid, 256, 0, st>>>(v1, key_rel, ns, key_tot); count_launch();
    GS_CUDA(c, cudaGetLastError());
    b1 = cub_bytes;
    GS_CUDA(c, cub::DeviceRadixSort::SortPairs(cub_tmp, b1, key_tot, key_tmp, v1, v0, (int)ns, 0, 64, st));
    count_launch(kCubSortLaunches);
    // v0 = final order
    if (kk) {
      gs_ranked_site* dst = out;
      if (out_is_host) {
        GS_CUDA(c, dev_grow(&c->d_ranked, &c->ranked_cap, kk));
        dst = c->d_ranked;
      }
      k_emit<<<(unsigned)kk, 32, 0, st>>>(v0, kk, c->d_sites, d_hist, c->d_kd, c->d_ktot, dst); count_launch();
      GS_CUDA(c, cudaGetLastError());
      if (out_is_host)
        GS_CUDA(c, cudaMemcpyAsync(out, dst, kk * sizeof(gs_ranked_site), cudaMemcpyDeviceToHost, st));
    }
  }
  GS_CUDA(c, cudaStreamSynchronize(st));
  if (n_out) *n_out = kk;
  return GS_OK;
}

void rank_free(gs_ctx* c) {
  for (int b = 0; b < 2; b++) {
    if (c->d_rank_keys[b]) cudaFree(c->d_rank_keys[b]);
    if (c->d_rank_vals[b]) cudaFree(c->d_rank_vals[b]);
    c->d_rank_keys[b] = nullptr;
    c->d_rank_vals[b] = nullptr;
  }
  if (c->d_sort_tmp) cudaFree(c->d_sort_tmp);
  if (c->d_ktot) cudaFree(c->d_ktot);
  if (c->d_ranked) cudaFree(c->d_ranked);
  c->d_sort_tmp = nullptr;
  c->d_ktot = nullptr;
  c->d_ranked = nullptr;
  c->rank_cap = 0;
  c->sort_tmp_bytes = 0;
  c->ranked_cap = 0;
}

}  // namespace gs
