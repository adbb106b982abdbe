// ctx.h — the library context (opaque gs_ctx behind the C ABI) and internal launch helpers.
#pragma once
#include <cuda_runtime.h>

#include <string>
#include <unordered_map>
#include <vector>

#include "../../include/gpuscout_b200.h"
#include "record.h"

namespace gs {

// instructions per detection window (never crosses a kernel): 256, or 1024 for modules of at least
// kBigModule instructions (fewer, longer windows: smaller carry tables; a small module needs the
// short windows to fill the GPU with warps)
#ifndef GS_WIN_SMALL
#define GS_WIN_SMALL 256
#endif
constexpr uint32_t kWinSmall = GS_WIN_SMALL, kWinBig = 1024;
constexpr uint64_t kBigModule = 16ull << 20;

// A device buffer that only grows; freed with the context.
struct DevBuf {
  void* p = nullptr;
  size_t bytes = 0;
};

// Candidate arrays: one entry per traced memory instruction or conversion.
struct CandArrays {
  uint32_t *idx = nullptr, *kernel = nullptr, *base_rd = nullptr, *data_rd = nullptr, *tv = nullptr,
           *grp = nullptr,
           *cont = nullptr;  // a trace left its window: the RD value to resume from (tk = kTCont, tv = register)
  uint8_t *ld = nullptr, *tk = nullptr, *depth = nullptr, *flags = nullptr;
  Rec* rec = nullptr;  // the candidate's instruction record (later passes read it coalesced, not gathered)
  uint32_t* chain4 = nullptr;  // the first kChain4 chain elements of the trace (k_write re-traces longer ones)
  unsigned long long* choff = nullptr;  // chain offsets (exclusive scan of chain lengths)
};

// Key-group statistics of global loads (R3), their distinct offsets, and the store roots (R8),
// as open-addressing hash tables partitioned by kernel: kernel k owns a power-of-two region of each
// table sized to twice its global loads / stores. Candidates are traced in instruction order, so
// the regions the resident threads update at any time are a few kernels' worth and stay in L2
// (one table over the whole module sent every update to a random DRAM sector).
struct KHash {
  unsigned long long gofs, rofs;  // first entry of the kernel's group / root region
  uint32_t gmask, rmask;          // region size - 1 (power of two)
  uint32_t pad[2];
};
struct GEnt {  // one 32-byte sector per group
  unsigned long long key;
  uint32_t nload, n32, nall;
  int32_t mn, mx;
  uint32_t bits;  // bits 0-1: OR of (offset & 3); bits 2-3: AND of (offset & 3)
};
struct OEnt {  // a (group slot, offset) pair; flags: 1 = seen as a 32-bit load, 2 = seen
  unsigned long long key;
  uint32_t flags, pad;
};
struct GroupTable {
  uint64_t gtot = 0, rtot = 0;  // entries of the group / offset tables and of the root table
  GEnt* g = nullptr;
  OEnt* o = nullptr;            // the offset table shares the group table's regions
  unsigned long long* r = nullptr;
  KHash* kh = nullptr;
};

}  // namespace gs

struct gs_ctx {
  int device = 0;
  cudaStream_t stream = nullptr;
  gs_config cfg{};
  std::string err;

  // ---- loaded SASS (host mirrors)
  bool loaded = false;
  uint32_t n_kernels = 0, n_win = 0;
  uint64_t n_instr = 0, n_cand = 0, n_ldg = 0, n_store = 0;
  std::vector<std::string> names;
  std::vector<gs::KDesc> kd_h;
  std::vector<gs::WDesc> wd_h;
  std::vector<uint32_t> cbase_h;  // candidate base per window (n_win + 1)
  std::vector<int32_t> lines_h;
  uint32_t n_lgroups = 0;             // source-line groups (kernel, file, line), 0 without line info
  std::vector<uint32_t> use_off_h;     // register-pressure inputs (R36), uploaded on first use:
  std::vector<uint8_t> use_reg_h;      //   GPR uses per slot (CSR, global offsets), branch targets
  uint32_t win = gs::kWinSmall;        // detection window length of the loaded module
  std::vector<int32_t> tgt_h;          //   (kernel-local index, -1 none, -2 - x indirect-branch list x)
  std::vector<uint32_t> xoff_h;        // indirect-branch successor lists (R38i, CSR over x)
  std::vector<int32_t> xtgt_h;

  // ---- device copies
  gs::Rec* d_rec = nullptr;
  gs::KDesc* d_kd = nullptr;
  gs::WDesc* d_wd = nullptr;
  uint32_t* d_cbase = nullptr;
  uint32_t* d_lgrp = nullptr;   // per slot: its source-line group, ~0u if none (only when n_lgroups)
  uint32_t* d_goff = nullptr;   // group -> first entry of d_gslot (n_lgroups + 1)
  uint32_t* d_gslot = nullptr;  // slots ordered by group
  uint32_t* d_use_off = nullptr;  // register pressure inputs on the device (lazy)
  uint8_t* d_use_reg = nullptr;
  int32_t* d_tgt = nullptr;
  uint32_t* d_xoff = nullptr;
  int32_t* d_xtgt = nullptr;
  void* d_lv = nullptr;           // liveness scratch
  size_t lv_bytes = 0;

  // ---- detection scratch
  uint32_t* d_tab = nullptr;  // n_win x 320 last-writer summaries -> carry-in tables
  int32_t* d_ldiff = nullptr; // loop-event difference array (kept zero between calls)
  int32_t* d_wsum = nullptr;  // per-window loop-event sum
  int32_t* d_wloop = nullptr; // per-window loop-depth carry-in
  uint32_t* d_wev = nullptr;  // per-window loop-event count
  uint32_t* d_ptrrd = nullptr;  // RD of each instruction's pointer operand (idx+1, 0 = ENTRY)
  uint32_t* d_narith = nullptr; // n_arith per global load (sparse)
  gs::CandArrays cand;
  gs::GroupTable grp;
  std::vector<gs::KHash> kh_h;
  gs_kernel_stats* d_kstats = nullptr;
  std::vector<gs_kernel_stats> kstats_h;
  void* d_scan_tmp = nullptr;
  size_t scan_tmp_bytes = 0;

  // ---- detection result
  bool detected = false;
  uint32_t det_kb = 0, det_ke = 0;
  uint64_t det_c0 = 0, det_c1 = 0;
  gs_site* d_sites = nullptr;
  uint64_t sites_cap = 0, n_sites = 0;
  uint32_t* d_chain = nullptr;
  uint64_t chain_cap = 0, n_chain = 0;

  // ---- attribution / ranking scratch
  int last_hist_mode = 0, last_hist_bits = 0;
  uint32_t last_hist_table_words = 0;  // WINDOW table size of the last histogram launch
  void* d_part = nullptr;              // PARTITION scratch: counts, bucket starts, partitioned copy
  size_t part_bytes = 0;
  unsigned long long* d_tileq = nullptr;  // WINDOW histogram work-stealing queue
  uint64_t tileq_cap = 0;
  uint32_t* d_defer = nullptr;  // WINDOW histogram: per-CTA rings of deferred (out-of-window) samples
  uint64_t defer_cap = 0;
  unsigned long long* d_rank_keys[2] = {nullptr, nullptr};
  uint32_t* d_rank_vals[2] = {nullptr, nullptr};
  uint64_t rank_cap = 0;
  int rank_bits_guess[2] = {-1, -1};  // bit widths of max(rel), max(tot) used by the last rank call
  cudaGraphExec_t det_exec = nullptr;   // the detection sequence as a CUDA graph (see detect_run)
  std::vector<uintptr_t> det_key;
  uint64_t det_graph_launches = 0;
  cudaGraphExec_t rank_exec = nullptr;  // the rank sequence as a CUDA graph, replayed while its key repeats
  std::vector<uintptr_t> rank_key;
  uint64_t rank_graph_launches = 0;
  void* d_sort_tmp = nullptr;
  size_t sort_tmp_bytes = 0;
  // CUPTI ingest (cupti.cpp, R39): stall-reason index -> reason id (-2 skipped, -1 unknown), kernel
  // name -> index of the loaded module, pinned staging + device copy of the flattened records
  std::unordered_map<uint32_t, int> cupti_reason;
  std::unordered_map<std::string, uint32_t> kernel_index;
  void* h_cupti = nullptr;
  void* d_cupti = nullptr;
  uint64_t cupti_cap = 0;
  unsigned long long* d_ktot = nullptr;
  uint64_t ktot_cap = 0;
  gs_ranked_site* d_ranked = nullptr;
  uint32_t* d_jrow = nullptr;   // GS_JOIN_LINE / GS_JOIN_CONSUMER: joined row per site (32 u32, saturated)
  // GS_JOIN_CONSUMER (R37), built by gs_detect: per GPR use its defining slot, and per slot the
  // group {slot, its consumers} (CSR over global slots, valid for the detected kernels)
  uint32_t* d_cdef = nullptr;   // per use (global use index): def slot or ~0u
  uint64_t cdef_cap = 0;
  uint32_t* d_ccnt = nullptr;   // per slot (+1): 1 + consumers
  uint64_t ccnt_cap = 0;
  uint32_t* d_cgoff = nullptr;  // per slot (+1): first entry of d_cgslot
  uint64_t cgoff_cap = 0;
  uint32_t* d_cgslot = nullptr; // the slot itself, then its consumers
  uint64_t cgslot_cap = 0;
  unsigned long long* d_ctot = nullptr;
  bool cons_ready = false;      // the consumer groups belong to the current detection
  uint64_t jrow_cap = 0;
  uint64_t ranked_cap = 0;
  void* h_pin = nullptr;  // pinned host scratch for small D2H results (async copies, no hidden sync)
  size_t h_pin_bytes = 0;
  // detection's own pinned results (totals + per-kernel counters): an asynchronous gs_detect
  // (n_sites == NULL) leaves them in flight until detect_finish
  void* h_det = nullptr;
  size_t h_det_bytes = 0;
  bool det_pending = false;
  uint64_t det_nc = 0;
  uint32_t det_D = 0;
  uint32_t* h_stage[2] = {nullptr, nullptr};  // pinned staging for host sample input
  uint32_t* d_stage[2] = {nullptr, nullptr};
  cudaEvent_t ev_stage[2] = {nullptr, nullptr};   // histogram of staging buffer b done (ctx stream)
  cudaEvent_t ev_copied[2] = {nullptr, nullptr};  // H2D into staging buffer b done (copy stream)
  cudaStream_t copy_stream = nullptr;             // host input: H2D copies overlap the histogram
  // detection: hash-table zeroing on a side stream, forked from and joined into the context's stream
  cudaStream_t side_stream = nullptr;
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
  // GPU time of the last device-input gs_attribute_samples (events around its enqueued work)
  cudaEvent_t ev_pass[2] = {nullptr, nullptr};
  bool pass_timed = false;
  int dev_sms = 0;                   // cached multiprocessor count
  int cluster_sort_ok = -1;          // rank: 16-CTA cluster sort usable (-1: not probed yet)
  const void* smem_fn[4] = {nullptr, nullptr, nullptr, nullptr};  // kernels whose dynamic smem limit
  size_t smem_set[4] = {0, 0, 0, 0};                               // was raised, and to what
  size_t stage_words = 0;
};

namespace gs {

// process-wide launch counter (gs_launch_count)
void count_launch(uint64_t n = 1);
void count_launch_undo(uint64_t n);
uint64_t launch_count_now();

// error helpers (set ctx->err, return status)
gs_status fail(gs_ctx* c, gs_status s, const std::string& msg);
gs_status cuda_fail(gs_ctx* c, cudaError_t e, const char* what);
#define GS_CUDA(ctx, call)                                  \
  do {                                                      \
    cudaError_t e_ = (call);                                \
    if (e_ != cudaSuccess) return gs::cuda_fail(ctx, e_, #call); \
  } while (0)

// pinned host scratch of at least `bytes` (contents not preserved)
inline cudaError_t pin_grow(gs_ctx* c, size_t bytes) {
  if (c->h_pin && c->h_pin_bytes >= bytes) return cudaSuccess;
  if (c->h_pin) cudaFreeHost(c->h_pin);
  c->h_pin = nullptr;
  c->h_pin_bytes = 0;
  cudaError_t e = cudaHostAlloc(&c->h_pin, bytes < 4096 ? 4096 : bytes, cudaHostAllocDefault);
  if (e == cudaSuccess) c->h_pin_bytes = bytes < 4096 ? 4096 : bytes;
  return e;
}

template <typename T>
cudaError_t dev_grow(T** p, uint64_t* cap, uint64_t need) {
  if (*p && *cap >= need) return cudaSuccess;
  if (*p) cudaFree(*p);
  *p = nullptr;
  *cap = 0;
  if (need == 0) return cudaSuccess;
  cudaError_t e = cudaMalloc((void**)p, need * sizeof(T));
  if (e == cudaSuccess) *cap = need;
  return e;
}

// launchers implemented in detect.cu / attrib.cu / rank.cu
gs_status detect_run(gs_ctx* c, uint32_t kb, uint32_t ke, uint64_t* n_sites);
gs_status detect_finish(gs_ctx* c);  // completes an asynchronous gs_detect (no-op otherwise)
gs_status detect_alloc(gs_ctx* c);  // after a load
void detect_free(gs_ctx* c);
gs_status pack_samples_run(gs_ctx* c, const uint32_t* d_raw, uint64_t n, uint32_t* d_words,
                           unsigned long long* d_n_invalid);
gs_status counts8_run(gs_ctx* c, const void* d_recs, uint64_t n, int32_t* d_hist, unsigned long long* d_n_invalid,
                      int accumulate);  // {compact bin, count} records
gs_status counts_run(gs_ctx* c, const uint32_t* d_recs, uint64_t n, int32_t* d_hist, unsigned long long* d_n_invalid,
                     int accumulate);
gs_status hist_run(gs_ctx* c, const uint32_t* d_words, uint64_t n, int32_t* d_hist,
                   unsigned long long* d_n_invalid, int accumulate, bool zero_first);
// d_hist holds the rows of slots [slot0, ...) (row width cfg.hist_row)
gs_status rank_run(gs_ctx* c, const int32_t* d_hist, uint32_t slot0, uint64_t k, gs_ranked_site* out,
                   bool out_is_host, uint64_t* n_out);
void attrib_free(gs_ctx* c);
gs_status liveness_run(gs_ctx* c, uint32_t kb, uint32_t ke, uint16_t* d_live);
// upload the packer's GPR use lists and branch targets (once per gs_load_sass)
gs_status uses_upload(gs_ctx* c);
void liveness_free(gs_ctx* c);
void rank_free(gs_ctx* c);
void rank_reset_graph(gs_ctx* c);
gs_status cupti_reasons(gs_ctx* c, size_t n, const uint32_t* index, const char* const* names);
gs_status cupti_run(gs_ctx* c, const void* pc_data, size_t n, uint64_t crc, int32_t* d_hist,
                    unsigned long long* d_n_invalid, int accumulate, unsigned long long* n_skipped,
                    unsigned long long* n_records);
cudaError_t cupti_grow(gs_ctx* c, uint64_t n);
void cupti_free(gs_ctx* c);

// device-wide exclusive scan of u32 counts into u32 or u64 offsets; total written to *d_total
gs_status scan_u32(gs_ctx* c, const uint32_t* in, uint32_t* out, uint64_t n, unsigned long long* d_total);
gs_status scan_u32_to_u64(gs_ctx* c, const uint32_t* in, unsigned long long* out, uint64_t n,
                          unsigned long long* d_total);

}  // namespace gs
