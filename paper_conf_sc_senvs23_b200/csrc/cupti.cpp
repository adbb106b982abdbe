// cupti.cpp — CUPTI PC-sampling ingest (§2.2, [probe 8]; R39).
//
// CUPTI delivers PC samples already aggregated per PC: CUpti_PCSamplingPCData {cubinCrc, pcOffset,
// functionName, stallReason[] = {CUPTI stall-reason index, samples}} in host memory (the names and
// the per-reason arrays are host pointers). The stall-reason indices are CUPTI's own; their names
// ("smsp__pcsamp_warps_issue_stalled_<reason>[_not_issued]") come from
// cuptiPCSamplingGetStallReasons and are handed to gs_cupti_stall_reasons once.
//
// Host side (this file): the records are flattened, in parallel over record ranges, into {kernel,
// pc, reason, count} count records (kernel by function name among the loaded module's kernels,
// reason by name among the 19 ncu reasons; a "_not_issued" counter is a subset of the same
// samples and is skipped; a foreign cubin, an unknown function or reason: kernel = invalid).
// Device side: one pinned staging copy and the weighted scatter-add k_counts of
// gs_attribute_counts (attrib.cu), which also counts the invalid weight.
#include <cupti_pcsampling.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

#include "ctx.h"

namespace gs {

static_assert(sizeof(CUpti_PCSamplingPCData) == 64, "CUPTI 12.9 PC record layout");
static_assert(sizeof(CUpti_PCSamplingStallReason) == 8, "CUPTI 12.9 stall reason layout");

namespace {
// the 19 reasons in id order (R17, SURVEY [probe 9])
const char* const kReasons[19] = {"barrier", "branch_resolving", "dispatch_stall", "drain", "imc_miss",
                                  "lg_throttle", "long_scoreboard", "math_pipe_throttle", "membar", "mio_throttle",
                                  "misc", "no_instructions", "not_selected", "selected", "short_scoreboard",
                                  "sleeping", "tex_throttle", "wait", "warpgroup_arrive"};
constexpr int kSkip = -2, kUnknown = -1;
constexpr uint32_t kBadKernel = 0xffffffffu;

int reason_of(const char* name) {
  static const char prefix[] = "smsp__pcsamp_warps_issue_stalled_";
  static const char ni[] = "_not_issued";
  const size_t n = strlen(name), np = sizeof(prefix) - 1, nn = sizeof(ni) - 1;
  if (n <= np || memcmp(name, prefix, np) != 0) return kUnknown;
  if (n > np + nn && memcmp(name + n - nn, ni, nn) == 0) return kSkip;
  for (int r = 0; r < 19; r++)
    if (strcmp(name + np, kReasons[r]) == 0) return r;
  return kUnknown;
}
}  // namespace

gs_status cupti_reasons(gs_ctx* c, size_t n, const uint32_t* index, const char* const* names) {
  c->cupti_reason.clear();
  for (size_t i = 0; i < n; i++) {
    if (!names[i]) return fail(c, GS_E_INVAL, "null stall-reason name");
    c->cupti_reason[index[i]] = reason_of(names[i]);
  }
  return GS_OK;
}

gs_status cupti_run(gs_ctx* c, const void* pc_data, size_t n, uint64_t crc, int32_t* d_hist,
                    unsigned long long* d_n_invalid, int accumulate, unsigned long long* n_skipped,
                    unsigned long long* n_records) {
  const CUpti_PCSamplingPCData* pcs = static_cast<const CUpti_PCSamplingPCData*>(pc_data);
  if (c->kernel_index.empty() && c->n_kernels) {
    c->kernel_index.reserve(c->n_kernels * 2);
    for (uint32_t k = 0; k < c->n_kernels; k++) c->kernel_index.emplace(c->names[k], k);
  }
  // pass 1 (parallel): entries per record range; then two flattening phases (each thread the first,
  // then the second half of its range): the H2D copy and the scatter-add of phase 0's records run
  // while phase 1 flattens
  const int nt = (int)std::max<size_t>(1, std::min<size_t>({16, std::thread::hardware_concurrency(), n / 4096 + 1}));
  constexpr int kPh = 2;
  std::vector<uint64_t> cnt(kPh * nt + 1, 0);  // entries of (phase, thread) in phase-major order
  std::vector<unsigned long long> skipped(nt, 0);
  auto range = [&](int ph, int t, size_t* a, size_t* b) {
    const size_t ta = n * t / nt, tb = n * (t + 1) / nt, tm = ta + (tb - ta) / 2;
    *a = ph ? tm : ta;
    *b = ph ? tb : tm;
  };
  auto run = [&](auto fn) {
    std::vector<std::thread> th;
    for (int t = 1; t < nt; t++) th.emplace_back(fn, t);
    fn(0);
    for (auto& x : th) x.join();
  };
  run([&](int t) {
    for (int ph = 0; ph < kPh; ph++) {
      size_t a, b;
      range(ph, t, &a, &b);
      uint64_t m = 0;
      for (size_t i = a; i < b; i++) m += pcs[i].stallReasonCount;
      cnt[ph * nt + t + 1] = m;
    }
  });
  for (int q = 0; q < kPh * nt; q++) cnt[q + 1] += cnt[q];
  const uint64_t total = cnt[kPh * nt];
  if (n_records) *n_records = total;
  GS_CUDA(c, cupti_grow(c, total));
  // flattened records {compact bin, count} (8 B: half the H2D bytes of {kernel, pc, reason, count});
  // validation here (R30): unknown kernel or reason, misaligned or out-of-range pc -> bin ~0u
  uint2* h = static_cast<uint2*>(c->h_cupti);
  const uint32_t nr = c->cfg.n_reasons;
  // stall-reason index -> reason as a flat table (a hash lookup per entry was most of the host time)
  uint32_t max_idx = 0;
  for (const auto& kv : c->cupti_reason) max_idx = std::max(max_idx, kv.first);
  std::vector<int> rtab(c->cupti_reason.empty() ? 0 : (size_t)max_idx + 1, kUnknown);
  for (const auto& kv : c->cupti_reason) rtab[kv.first] = kv.second;
  cudaStream_t st = c->stream;
  if (!accumulate && c->n_instr) GS_CUDA(c, cudaMemsetAsync(d_hist, 0, c->n_instr * c->cfg.hist_row * 4, st));
  for (int ph = 0; ph < kPh; ph++) {
  run([&](int t) {
    size_t a, b;
    range(ph, t, &a, &b);
    uint64_t o = cnt[ph * nt + t];
    unsigned long long sk = 0;
    // CUPTI hands out one name pointer per function: consecutive records of a function share it,
    // so the (string-keyed) kernel lookup runs once per run of records, and once per pointer
    std::unordered_map<const char*, uint32_t> by_ptr;
    const char* last_name = nullptr;
    uint32_t last_k = kBadKernel;
    for (size_t i = a; i < b; i++) {
      const CUpti_PCSamplingPCData& d = pcs[i];
      uint32_t k = kBadKernel;
      if (d.functionName && (crc == 0 || d.cubinCrc == crc) && d.pcOffset <= 0xffffffffull) {
        if (d.functionName != last_name) {
          auto pit = by_ptr.find(d.functionName);
          if (pit != by_ptr.end()) {
            last_k = pit->second;
          } else {
            auto it = c->kernel_index.find(d.functionName);
            last_k = it != c->kernel_index.end() ? it->second : kBadKernel;
            by_ptr.emplace(d.functionName, last_k);
          }
          last_name = d.functionName;
        }
        k = last_k;
      }
      // the record's first compact bin (reason 0) when its kernel and pc are valid, else ~0u
      uint32_t kbin = 0xffffffffu;
      if (k != kBadKernel && (d.pcOffset & 15u) == 0) {
        const KDesc& K = c->kd_h[k];
        const uint64_t pcs16 = d.pcOffset >> 4;
        if (pcs16 < K.n) kbin = (K.first + (uint32_t)pcs16) * nr;
      }
      for (size_t q = 0; q < d.stallReasonCount; q++) {
        const CUpti_PCSamplingStallReason& e = d.stallReason[q];
        const uint32_t ri = e.pcSamplingStallReasonIndex;
        const int r = ri < rtab.size() ? rtab[ri] : kUnknown;
        if (r == kSkip) {  // a subset of the same samples (R39): not attributed, not invalid
          sk += e.samples;
          h[o++] = make_uint2(0u, 0u);  // a zero-weight record keeps the layout fixed
          continue;
        }
        h[o++] = make_uint2(kbin != 0xffffffffu && r >= 0 && (uint32_t)r < nr ? kbin + (uint32_t)r : 0xffffffffu, e.samples);
      }
    }
    skipped[t] += sk;
  });
    // this phase's records: copy and scatter-add (async) while the next phase flattens
    const uint64_t p0 = cnt[ph * nt], p1 = cnt[(ph + 1) * nt];
    if (p1 > p0) {
      GS_CUDA(c, cudaMemcpyAsync(static_cast<uint2*>(c->d_cupti) + p0, h + p0, (p1 - p0) * 8, cudaMemcpyHostToDevice,
                                 st));
      const gs_status s = counts8_run(c, static_cast<uint2*>(c->d_cupti) + p0, p1 - p0, d_hist, d_n_invalid, 1);
      if (s != GS_OK) return s;
    }
  }
  unsigned long long sk = 0;
  for (auto v : skipped) sk += v;
  if (n_skipped) *n_skipped = sk;
  // the staging buffer is reused by the next call: wait for this copy (the scatter-add stays async)
  GS_CUDA(c, cudaStreamSynchronize(st));
  return GS_OK;
}

cudaError_t cupti_grow(gs_ctx* c, uint64_t n) {
  if (c->cupti_cap >= n && c->h_cupti) return cudaSuccess;
  if (c->h_cupti) cudaFreeHost(c->h_cupti);
  if (c->d_cupti) cudaFree(c->d_cupti);
  c->h_cupti = nullptr;
  c->d_cupti = nullptr;
  c->cupti_cap = 0;
  const uint64_t cap = std::max<uint64_t>(n, 4096);
  cudaError_t e = cudaHostAlloc(&c->h_cupti, cap * 16, cudaHostAllocDefault);
  if (e != cudaSuccess) return e;
  e = cudaMalloc(&c->d_cupti, cap * 16);
  if (e != cudaSuccess) return e;
  c->cupti_cap = cap;
  return cudaSuccess;
}

void cupti_free(gs_ctx* c) {
  if (c->h_cupti) cudaFreeHost(c->h_cupti);
  if (c->d_cupti) cudaFree(c->d_cupti);
  c->h_cupti = nullptr;
  c->d_cupti = nullptr;
  c->cupti_cap = 0;
}

}  // namespace gs
