// api.cu — the C ABI (include/gpuscout_b200.h): context, SASS loading, entry points.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>
#include <thread>

#include "ctx.h"
#include "loader.h"

#include <atomic>

namespace gs {

static std::atomic<uint64_t> g_launches{0};
void count_launch(uint64_t n) { g_launches.fetch_add(n, std::memory_order_relaxed); }
void count_launch_undo(uint64_t n) { g_launches.fetch_sub(n, std::memory_order_relaxed); }
uint64_t launch_count_now() { return g_launches.load(std::memory_order_relaxed); }

gs_status fail(gs_ctx* c, gs_status s, const std::string& msg) {
  if (c) c->err = msg;
  return s;
}
gs_status cuda_fail(gs_ctx* c, cudaError_t e, const char* what) {
  return fail(c, GS_E_CUDA, std::string(what) + ": " + cudaGetErrorString(e));
}

namespace {

uint64_t pow2_ceil(uint64_t n) {
  uint64_t c = 1;
  while (c < n) c <<= 1;
  return c;
}

void free_loaded(gs_ctx* c) {
  detect_free(c);
  rank_reset_graph(c);
  c->kernel_index.clear();
  if (c->d_rec) cudaFree(c->d_rec);
  if (c->d_kd) cudaFree(c->d_kd);
  if (c->d_wd) cudaFree(c->d_wd);
  if (c->d_cbase) cudaFree(c->d_cbase);
  if (c->d_lgrp) cudaFree(c->d_lgrp);
  if (c->d_goff) cudaFree(c->d_goff);
  if (c->d_gslot) cudaFree(c->d_gslot);
  c->d_lgrp = c->d_goff = c->d_gslot = nullptr;
  liveness_free(c);
  c->n_lgroups = 0;
  c->d_rec = nullptr;
  c->d_kd = nullptr;
  c->d_wd = nullptr;
  c->d_cbase = nullptr;
  c->loaded = false;
}

bool is_device_ptr(const void* p) {
  cudaPointerAttributes a;
  if (cudaPointerGetAttributes(&a, p) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return a.type == cudaMemoryTypeDevice || a.type == cudaMemoryTypeManaged;
}

}  // namespace
}  // namespace gs

using namespace gs;

extern "C" {

const char* gs_version(void) { return "gpuscout_b200 0.1 (sm_100a)"; }

gs_status gs_create(gs_ctx** out, int device, void* cuda_stream, const gs_config* cfg) {
  if (!out) return GS_E_INVAL;
  *out = nullptr;
  gs_ctx* c = new (std::nothrow) gs_ctx();
  if (!c) return GS_E_NOMEM;
  c->device = device;
  c->stream = static_cast<cudaStream_t>(cuda_stream);
  if (cfg) c->cfg = *cfg;
  if (!c->cfg.trace_depth) c->cfg.trace_depth = 64;
  if (!c->cfg.n_reasons) c->cfg.n_reasons = 19;
  if (!c->cfg.shmem_min_arith) c->cfg.shmem_min_arith = 1;
  if (!c->cfg.shmem_min_loads) c->cfg.shmem_min_loads = 2;
  if (!c->cfg.hist_row) c->cfg.hist_row = 32;
  if (c->cfg.trace_depth > 255 || c->cfg.n_reasons > 32 || c->cfg.hist_mode > GS_HIST_PARTITION ||
      (c->cfg.hist_row != 32 && c->cfg.hist_row != c->cfg.n_reasons) || c->cfg.join_mode > GS_JOIN_CONSUMER ||
      (c->cfg.hist_counter_bits != 0 && c->cfg.hist_counter_bits != 16 && c->cfg.hist_counter_bits != 32)) {
    delete c;
    return GS_E_INVAL;
  }
  cudaError_t e = cudaSetDevice(device);
  if (e != cudaSuccess) {
    delete c;
    return GS_E_CUDA;
  }
  *out = c;
  return GS_OK;
}

void gs_destroy(gs_ctx* c) {
  if (!c) return;
  cudaSetDevice(c->device);
  if (c->stream) cudaStreamSynchronize(c->stream);
  else cudaDeviceSynchronize();
  free_loaded(c);
  attrib_free(c);
  rank_free(c);
  cupti_free(c);
  if (c->h_pin) cudaFreeHost(c->h_pin);
  if (c->h_det) cudaFreeHost(c->h_det);
  if (c->side_stream) {
    cudaStreamSynchronize(c->side_stream);
    cudaStreamDestroy(c->side_stream);
  }
  if (c->ev_fork) cudaEventDestroy(c->ev_fork);
  if (c->ev_join) cudaEventDestroy(c->ev_join);
  delete c;
}

const char* gs_last_error(const gs_ctx* c) { return c ? c->err.c_str() : "null context"; }

gs_status gs_load_sass(gs_ctx* c, const char* text, size_t len, uint32_t* n_kernels, uint64_t* n_instr) {
  if (!c || (!text && len)) return fail(c, GS_E_INVAL, "null argument");
  c->err.clear();
  GS_CUDA(c, cudaSetDevice(c->device));
  std::vector<ParsedKernel> ks;
  std::string err;
  const int nt = (int)std::max(1u, std::min(16u, std::thread::hardware_concurrency()));
  // GS_TIMING=1: host phase times of the load on stderr (parse | pack tables | upload | scratch)
  static const bool timing = getenv("GS_TIMING") != nullptr;
  using clk = std::chrono::steady_clock;
  const auto t0 = clk::now();
  if (!parse_sass(text, len, nt, &ks, &err)) return fail(c, GS_E_PARSE, err);
  const auto t1 = clk::now();
  uint64_t P = 0;
  for (auto& k : ks) P += k.recs.size();
  if (P > 0x7ffffffeull) return fail(c, GS_E_RANGE, "more than 2^31-2 instructions");
  if (c->stream) GS_CUDA(c, cudaStreamSynchronize(c->stream));
  free_loaded(c);
  c->n_kernels = (uint32_t)ks.size();
  c->n_instr = P;
  c->win = P >= kBigModule ? kWinBig : kWinSmall;
  c->names.clear();
  c->kd_h.assign(ks.size(), KDesc{});
  c->wd_h.clear();
  c->lines_h.clear();
  c->lines_h.reserve(P);
  c->cbase_h.clear();
  c->use_off_h.assign(1, 0);
  c->use_reg_h.clear();
  c->tgt_h.clear();
  c->xoff_h.assign(1, 0);
  c->xtgt_h.clear();
  c->n_cand = c->n_ldg = c->n_store = 0;
  c->kh_h.assign(ks.size(), KHash{});
  c->grp.gtot = c->grp.rtot = 0;
  // per-kernel offsets (sequential, O(kernels)), then the kernels' records and tables are copied
  // into the module arrays in parallel
  const size_t K = ks.size();
  std::vector<uint64_t> use_base(K + 1, 0), xl_base(K + 1, 0), xt_base(K + 1, 0);
  uint32_t slot = 0, nwin = 0;
  for (size_t k = 0; k < K; k++) {
    const ParsedKernel& pk = ks[k];
    KDesc& Kd = c->kd_h[k];
    Kd.first = slot;
    Kd.n = (uint32_t)pk.recs.size();
    Kd.param_base = pk.param_base | (std::min<uint32_t>(pk.nregs, 255u) << 16);
    Kd.win0 = nwin;
    nwin += (Kd.n + c->win - 1) / c->win;
    slot += Kd.n;
    use_base[k + 1] = use_base[k] + pk.use_reg.size();
    xl_base[k + 1] = xl_base[k] + (pk.xtgt_off.empty() ? 0 : pk.xtgt_off.size() - 1);
    xt_base[k + 1] = xt_base[k] + pk.xtgt.size();
  }
  std::vector<Rec> recs(P);
  c->lines_h.resize(P);
  c->use_off_h.assign(P + 1, 0);
  c->use_reg_h.resize(use_base[K]);
  c->tgt_h.resize(P);
  c->xoff_h.assign(xl_base[K] + 1, 0);
  c->xtgt_h.resize(xt_base[K]);
  c->wd_h.resize(nwin);
  std::vector<uint32_t> wcand(nwin, 0);
  std::vector<uint64_t> kldg(K, 0), kst(K, 0);
  {
    std::atomic<size_t> next(0);
    auto fill = [&]() {
      for (;;) {
        const size_t k = next.fetch_add(1);
        if (k >= K) return;
        const ParsedKernel& pk = ks[k];
        const KDesc& Kd = c->kd_h[k];
        std::copy(pk.recs.begin(), pk.recs.end(), recs.begin() + Kd.first);
        std::copy(pk.lines.begin(), pk.lines.end(), c->lines_h.begin() + Kd.first);
        std::copy(pk.use_reg.begin(), pk.use_reg.end(), c->use_reg_h.begin() + use_base[k]);
        for (size_t i = 1; i < pk.use_off.size(); i++)  // register-pressure inputs, offsets made global
          c->use_off_h[Kd.first + i] = (uint32_t)(use_base[k] + pk.use_off[i]);
        const int32_t x0 = (int32_t)xl_base[k];  // indirect-branch lists: global list ids
        for (size_t i = 0; i < pk.tgt.size(); i++) {
          const int32_t t = pk.tgt[i];
          c->tgt_h[Kd.first + i] = t <= -2 ? t - x0 : t;
        }
        for (size_t x = 1; x < pk.xtgt_off.size(); x++)
          c->xoff_h[xl_base[k] + x] = (uint32_t)(xt_base[k] + pk.xtgt_off[x]);
        std::copy(pk.xtgt.begin(), pk.xtgt.end(), c->xtgt_h.begin() + xt_base[k]);
        uint64_t nl = 0, ns = 0;
        for (uint32_t s0 = 0, w = Kd.win0; s0 < Kd.n; s0 += c->win, w++) {
          const WDesc W{(uint32_t)k, Kd.first + s0, std::min(c->win, Kd.n - s0), 0};
          uint32_t nc = 0;
          for (uint32_t i = 0; i < W.len; i++) {  // candidates per window: static opcode classes
            const Rec& r = pk.recs[s0 + i];
            const uint32_t cls = op_class(r_op(r));
            if (cls & (C_TRACED | C_CONV)) nc++;
            if (r_op(r) == OP_LDG) nl++;
            if (cls & C_STORE) ns++;
          }
          c->wd_h[w] = W;
          wcand[w] = nc;
        }
        kldg[k] = nl;
        kst[k] = ns;
      }
    };
    std::vector<std::thread> th;
    for (int t = 1; t < nt; t++) th.emplace_back(fill);
    fill();
    for (auto& t : th) t.join();
  }
  c->cbase_h.resize(nwin);
  for (uint32_t w = 0; w < nwin; w++) {
    c->cbase_h[w] = (uint32_t)c->n_cand;
    c->n_cand += wcand[w];
  }
  for (size_t k = 0; k < K; k++) {  // the kernel's hash-table regions: a power of two >= 2x its loads / stores
    KHash& H = c->kh_h[k];
    const uint64_t gcap = pow2_ceil(2 * kldg[k] + 2), rcap = pow2_ceil(2 * kst[k] + 2);
    H.gofs = c->grp.gtot;
    H.rofs = c->grp.rtot;
    H.gmask = (uint32_t)(gcap - 1);
    H.rmask = (uint32_t)(rcap - 1);
    c->grp.gtot += gcap;
    c->grp.rtot += rcap;
    c->n_ldg += kldg[k];
    c->n_store += kst[k];
    c->names.push_back(std::move(ks[k].name));
  }
  c->cbase_h.push_back((uint32_t)c->n_cand);
  c->n_win = (uint32_t)c->wd_h.size();
  // source-line groups (R33): global id = kernel's base + kernel-local (file, line) key; CSR of slots
  std::vector<uint32_t> lgrp, goff, gslot;
  {
    uint64_t G = 0;
    for (auto& k : ks) G += k.n_lkeys;
    if (G) {
      lgrp.assign(P, ~0u);
      goff.assign(G + 1, 0);
      uint32_t gb = 0, sl = 0;
      for (auto& k : ks) {
        for (size_t i = 0; i < k.lkeys.size(); i++)
          if (k.lkeys[i] >= 0) { lgrp[sl + i] = gb + (uint32_t)k.lkeys[i]; goff[lgrp[sl + i] + 1]++; }
        gb += k.n_lkeys;
        sl += (uint32_t)k.recs.size();
      }
      for (uint64_t g = 0; g < G; g++) goff[g + 1] += goff[g];
      gslot.assign(goff[G], 0);
      std::vector<uint32_t> fill(goff.begin(), goff.end() - 1);
      for (uint32_t q = 0; q < P; q++)
        if (lgrp[q] != ~0u) gslot[fill[lgrp[q]]++] = q;
      c->n_lgroups = (uint32_t)G;
    }
  }
  if (c->n_cand > 0xffffffffull) return fail(c, GS_E_RANGE, "too many candidate instructions");
  GS_CUDA(c, cudaMalloc((void**)&c->d_rec, std::max<uint64_t>(P, 1) * sizeof(Rec)));
  GS_CUDA(c, cudaMalloc((void**)&c->d_kd, std::max<size_t>(ks.size(), 1) * sizeof(KDesc)));
  GS_CUDA(c, cudaMalloc((void**)&c->d_wd, std::max<size_t>(c->wd_h.size(), 1) * sizeof(WDesc)));
  GS_CUDA(c, cudaMalloc((void**)&c->d_cbase, c->cbase_h.size() * 4));
  const auto t2 = clk::now();
  if (P) GS_CUDA(c, cudaMemcpyAsync(c->d_rec, recs.data(), P * sizeof(Rec), cudaMemcpyHostToDevice, c->stream));
  if (!ks.empty())
    GS_CUDA(c, cudaMemcpyAsync(c->d_kd, c->kd_h.data(), ks.size() * sizeof(KDesc), cudaMemcpyHostToDevice, c->stream));
  if (!c->wd_h.empty())
    GS_CUDA(c, cudaMemcpyAsync(c->d_wd, c->wd_h.data(), c->wd_h.size() * sizeof(WDesc), cudaMemcpyHostToDevice,
                               c->stream));
  GS_CUDA(c, cudaMemcpyAsync(c->d_cbase, c->cbase_h.data(), c->cbase_h.size() * 4, cudaMemcpyHostToDevice, c->stream));
  if (c->n_lgroups) {
    GS_CUDA(c, cudaMalloc((void**)&c->d_lgrp, lgrp.size() * 4));
    GS_CUDA(c, cudaMalloc((void**)&c->d_goff, goff.size() * 4));
    GS_CUDA(c, cudaMalloc((void**)&c->d_gslot, std::max<size_t>(gslot.size(), 1) * 4));
    GS_CUDA(c, cudaMemcpyAsync(c->d_lgrp, lgrp.data(), lgrp.size() * 4, cudaMemcpyHostToDevice, c->stream));
    GS_CUDA(c, cudaMemcpyAsync(c->d_goff, goff.data(), goff.size() * 4, cudaMemcpyHostToDevice, c->stream));
    if (!gslot.empty())
      GS_CUDA(c, cudaMemcpyAsync(c->d_gslot, gslot.data(), gslot.size() * 4, cudaMemcpyHostToDevice, c->stream));
  }
  const auto t3 = clk::now();
  gs_status s = detect_alloc(c);
  if (s != GS_OK) return s;
  // pageable source buffers: wait for the copies before they go out of scope
  GS_CUDA(c, cudaStreamSynchronize(c->stream));
  if (timing) {
    const auto t4 = clk::now();
    const auto sec = [](clk::duration d) { return std::chrono::duration<double>(d).count(); };
    fprintf(stderr, "gs_load_sass: parse %.3f s, tables %.3f s, upload %.3f s, scratch+sync %.3f s (%u threads)\n",
            sec(t1 - t0), sec(t2 - t1), sec(t3 - t2), sec(t4 - t3), (unsigned)nt);
  }
  c->loaded = true;
  if (n_kernels) *n_kernels = c->n_kernels;
  if (n_instr) *n_instr = P;
  return GS_OK;
}

gs_status gs_kernel_table(const gs_ctx* c, uint32_t* first_slot, uint32_t* n_instr, size_t cap) {
  if (!c) return GS_E_INVAL;
  if (!c->loaded) return GS_E_STATE;
  const size_t n = std::min<size_t>(cap, c->n_kernels);
  for (size_t k = 0; k < n; k++) {
    if (first_slot) first_slot[k] = c->kd_h[k].first;
    if (n_instr) n_instr[k] = c->kd_h[k].n;
  }
  return GS_OK;
}

const char* gs_kernel_name(const gs_ctx* c, uint32_t k) {
  if (!c || !c->loaded || k >= c->n_kernels) return nullptr;
  return c->names[k].c_str();
}

gs_status gs_instr_lines(const gs_ctx* c, int32_t* lines, size_t cap) {
  if (!c || !lines) return GS_E_INVAL;
  if (!c->loaded) return GS_E_STATE;
  memcpy(lines, c->lines_h.data(), std::min<size_t>(cap, c->lines_h.size()) * 4);
  return GS_OK;
}

gs_status gs_detect(gs_ctx* c, uint32_t k_begin, uint32_t k_end, uint64_t* n_sites) {
  if (!c) return GS_E_INVAL;
  c->err.clear();
  if (!c->loaded) return fail(c, GS_E_STATE, "gs_detect before gs_load_sass");
  if (k_begin > k_end || k_end > c->n_kernels) return fail(c, GS_E_INVAL, "bad kernel range");
  GS_CUDA(c, cudaSetDevice(c->device));
  return detect_run(c, k_begin, k_end, n_sites);
}

gs_status gs_sites(const gs_ctx* c, const gs_site** d_sites, const uint32_t** d_chain, uint64_t* n_sites,
                   uint64_t* n_chain) {
  if (!c) return GS_E_INVAL;
  if (!c->detected) return GS_E_STATE;
  {
    const gs_status fs = detect_finish(const_cast<gs_ctx*>(c));  // an asynchronous gs_detect
    if (fs != GS_OK) return fs;
  }
  if (d_sites) *d_sites = c->d_sites;
  if (d_chain) *d_chain = c->d_chain;
  if (n_sites) *n_sites = c->n_sites;
  if (n_chain) *n_chain = c->n_chain;
  return GS_OK;
}

gs_status gs_sites_host(gs_ctx* c, gs_site* sites, size_t cap_sites, uint32_t* chain, size_t cap_chain) {
  if (!c) return GS_E_INVAL;
  if (!c->detected) return fail(c, GS_E_STATE, "gs_sites_host before gs_detect");
  GS_CUDA(c, cudaSetDevice(c->device));
  {
    const gs_status fs = detect_finish(c);
    if (fs != GS_OK) return fs;
  }
  const size_t ns = std::min<size_t>(cap_sites, c->n_sites), nch = std::min<size_t>(cap_chain, c->n_chain);
  if (sites && ns) GS_CUDA(c, cudaMemcpyAsync(sites, c->d_sites, ns * sizeof(gs_site), cudaMemcpyDeviceToHost, c->stream));
  if (chain && nch) GS_CUDA(c, cudaMemcpyAsync(chain, c->d_chain, nch * 4, cudaMemcpyDeviceToHost, c->stream));
  GS_CUDA(c, cudaStreamSynchronize(c->stream));
  return GS_OK;
}

gs_status gs_kernel_stats_get(const gs_ctx* c, gs_kernel_stats* out, size_t cap) {
  if (!c || !out) return GS_E_INVAL;
  if (!c->detected) return GS_E_STATE;
  {
    const gs_status fs = detect_finish(const_cast<gs_ctx*>(c));
    if (fs != GS_OK) return fs;
  }
  memcpy(out, c->kstats_h.data(), std::min<size_t>(cap, c->kstats_h.size()) * sizeof(gs_kernel_stats));
  return GS_OK;
}

gs_status gs_pack_samples(gs_ctx* c, const uint32_t* d_raw, uint64_t n, uint32_t* d_words,
                          unsigned long long* d_n_invalid) {
  if (!c || (n && (!d_raw || !d_words)) || !d_n_invalid) return fail(c, GS_E_INVAL, "null argument");
  c->err.clear();
  if (!c->loaded) return fail(c, GS_E_STATE, "gs_pack_samples before gs_load_sass");
  if (c->n_instr >= (1ull << 27)) return fail(c, GS_E_RANGE, "packed samples address at most 2^27 slots");
  GS_CUDA(c, cudaSetDevice(c->device));
  return pack_samples_run(c, d_raw, n, d_words, d_n_invalid);
}

gs_status gs_attribute_samples(gs_ctx* c, const uint32_t* samples, uint64_t n, int32_t* d_hist,
                               unsigned long long* d_n_invalid, int accumulate) {
  if (!c || (n && !samples) || !d_n_invalid) return fail(c, GS_E_INVAL, "null argument");
  c->err.clear();
  if (!c->loaded) return fail(c, GS_E_STATE, "gs_attribute_samples before gs_load_sass");
  if (!d_hist && c->n_instr) return fail(c, GS_E_INVAL, "null histogram");
  if (c->n_instr >= (1ull << 27)) return fail(c, GS_E_RANGE, "packed samples address at most 2^27 slots");
  GS_CUDA(c, cudaSetDevice(c->device));
  if (!n || is_device_ptr(samples)) {
    const gs_status hs = hist_run(c, samples, n, d_hist, d_n_invalid, accumulate, true);
    if (hs == GS_OK && c->ev_pass[1]) {  // hist_run recorded ev_pass[0] before its first enqueue
      GS_CUDA(c, cudaEventRecord(c->ev_pass[1], c->stream));
      c->pass_timed = true;
    }
    return hs;
  }
  // host input: chunks through two device staging buffers; the H2D copy of chunk i+1 runs on a
  // copy stream (copy engine) while the histogram of chunk i runs on the context's stream
#ifndef GS_STAGE_MWORDS
#define GS_STAGE_MWORDS 16
#endif
  const size_t chunk = size_t(GS_STAGE_MWORDS) << 20;  // words per staging buffer
  if (c->stage_words < chunk) {
    attrib_free(c);
    for (int b = 0; b < 2; b++) {
      GS_CUDA(c, cudaMalloc((void**)&c->d_stage[b], chunk * 4));
      GS_CUDA(c, cudaEventCreateWithFlags(&c->ev_stage[b], cudaEventDisableTiming));
      GS_CUDA(c, cudaEventCreateWithFlags(&c->ev_copied[b], cudaEventDisableTiming));
    }
    GS_CUDA(c, cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking));
    c->stage_words = chunk;
  }
  if (!accumulate) GS_CUDA(c, cudaMemsetAsync(d_hist, 0, c->n_instr * c->cfg.hist_row * 4, c->stream));
  // the copy stream starts after everything already enqueued on the context's stream
  GS_CUDA(c, cudaEventRecord(c->ev_stage[0], c->stream));
  GS_CUDA(c, cudaEventRecord(c->ev_stage[1], c->stream));
  uint64_t done = 0;
  int b = 0;
  while (done < n) {
    const uint64_t m = std::min<uint64_t>(chunk, n - done);
    GS_CUDA(c, cudaStreamWaitEvent(c->copy_stream, c->ev_stage[b], 0));  // buffer b free again
    GS_CUDA(c, cudaMemcpyAsync(c->d_stage[b], samples + done, m * 4, cudaMemcpyHostToDevice, c->copy_stream));
    GS_CUDA(c, cudaEventRecord(c->ev_copied[b], c->copy_stream));
    GS_CUDA(c, cudaStreamWaitEvent(c->stream, c->ev_copied[b], 0));
    gs_status s = hist_run(c, c->d_stage[b], m, d_hist, d_n_invalid, 1, false);
    if (s != GS_OK) return s;
    GS_CUDA(c, cudaEventRecord(c->ev_stage[b], c->stream));
    done += m;
    b ^= 1;
  }
  GS_CUDA(c, cudaStreamSynchronize(c->stream));
  return GS_OK;
}

gs_status gs_attribute_counts(gs_ctx* c, const uint32_t* d_recs, uint64_t n, int32_t* d_hist,
                              unsigned long long* d_n_invalid, int accumulate) {
  if (!c || (n && !d_recs) || !d_n_invalid) return fail(c, GS_E_INVAL, "null argument");
  c->err.clear();
  if (!c->loaded) return fail(c, GS_E_STATE, "gs_attribute_counts before gs_load_sass");
  if (!d_hist && c->n_instr) return fail(c, GS_E_INVAL, "null histogram");
  if (n && !is_device_ptr(d_recs)) return fail(c, GS_E_INVAL, "count records must be device memory");
  GS_CUDA(c, cudaSetDevice(c->device));
  return counts_run(c, d_recs, n, d_hist, d_n_invalid, accumulate);
}

gs_status gs_cupti_stall_reasons(gs_ctx* c, size_t n, const uint32_t* index, const char* const* names) {
  if (!c || (n && (!index || !names))) return fail(c, GS_E_INVAL, "null argument");
  c->err.clear();
  return cupti_reasons(c, n, index, names);
}

gs_status gs_attribute_cupti(gs_ctx* c, const void* pc_data, size_t n_pcs, uint64_t cubin_crc, int32_t* d_hist,
                             unsigned long long* d_n_invalid, int accumulate, unsigned long long* n_skipped,
                             unsigned long long* n_records) {
  if (!c || (n_pcs && !pc_data) || !d_n_invalid) return fail(c, GS_E_INVAL, "null argument");
  c->err.clear();
  if (!c->loaded) return fail(c, GS_E_STATE, "gs_attribute_cupti before gs_load_sass");
  if (!d_hist && c->n_instr) return fail(c, GS_E_INVAL, "null histogram");
  if (n_pcs && is_device_ptr(pc_data)) return fail(c, GS_E_INVAL, "CUPTI records must be host memory");
  GS_CUDA(c, cudaSetDevice(c->device));
  return cupti_run(c, pc_data, n_pcs, cubin_crc, d_hist, d_n_invalid, accumulate, n_skipped, n_records);
}

gs_status gs_register_pressure(gs_ctx* c, uint32_t k_begin, uint32_t k_end, uint16_t* d_live) {
  if (!c) return GS_E_INVAL;
  c->err.clear();
  if (!c->loaded) return fail(c, GS_E_STATE, "gs_register_pressure before gs_load_sass");
  if (k_begin > k_end || k_end > c->n_kernels) return fail(c, GS_E_INVAL, "bad kernel range");
  if (!d_live && k_end > k_begin) return fail(c, GS_E_INVAL, "null output");
  if (d_live && !is_device_ptr(d_live)) return fail(c, GS_E_INVAL, "output must be device memory");
  GS_CUDA(c, cudaSetDevice(c->device));
  return liveness_run(c, k_begin, k_end, d_live);
}

gs_status gs_rank_sites_slice(gs_ctx* c, const int32_t* d_hist, uint64_t slot_begin, uint64_t slot_end, uint64_t k,
                              gs_ranked_site* out, uint64_t* n_out) {
  if (!c) return GS_E_INVAL;
  c->err.clear();
  if (!c->detected) return fail(c, GS_E_STATE, "gs_rank_sites before gs_detect");
  {
    GS_CUDA(c, cudaSetDevice(c->device));
    const gs_status fs = detect_finish(c);
    if (fs != GS_OK) return fs;
  }
  if (slot_begin > slot_end || slot_end > c->n_instr) return fail(c, GS_E_INVAL, "bad slot range");
  if (!d_hist && slot_end > slot_begin) return fail(c, GS_E_INVAL, "null histogram");
  if (k && c->n_sites && !out) return fail(c, GS_E_INVAL, "null output");
  // the detected kernels' slots [first(kb), first(ke)) must lie inside the slice
  const uint64_t need0 = c->det_kb < c->n_kernels ? c->kd_h[c->det_kb].first : c->n_instr;
  const uint64_t need1 = c->det_ke < c->n_kernels ? c->kd_h[c->det_ke].first : c->n_instr;
  if (need1 > need0 && (slot_begin > need0 || slot_end < need1))
    return fail(c, GS_E_RANGE, "histogram slice [" + std::to_string(slot_begin) + ", " + std::to_string(slot_end) +
                                   ") does not cover the detected kernels' slots [" + std::to_string(need0) + ", " +
                                   std::to_string(need1) + ")");
  GS_CUDA(c, cudaSetDevice(c->device));
  const bool host = out ? !is_device_ptr(out) : true;
  return rank_run(c, d_hist, (uint32_t)slot_begin, k, out, host, n_out);
}

gs_status gs_rank_sites(gs_ctx* c, const int32_t* d_hist, uint64_t k, gs_ranked_site* out, uint64_t* n_out) {
  if (!c) return GS_E_INVAL;
  return gs_rank_sites_slice(c, d_hist, 0, c->n_instr, k, out, n_out);
}

uint64_t gs_launch_count(void) { return gs::g_launches.load(); }

int gs_last_hist_mode(const gs_ctx* c) { return c ? c->last_hist_mode : -1; }

gs_status gs_last_attribute_ms(gs_ctx* c, float* ms) {
  if (!c || !ms) return GS_E_INVAL;
  if (!c->pass_timed) return fail(c, GS_E_STATE, "no timed gs_attribute_samples call (device input) yet");
  GS_CUDA(c, cudaEventSynchronize(c->ev_pass[1]));
  GS_CUDA(c, cudaEventElapsedTime(ms, c->ev_pass[0], c->ev_pass[1]));
  return GS_OK;
}

}  // extern "C"
