/* gpuscout_b200.h — C ABI of the B200-native batched bottleneck-attribution library.
 *
 * Method: GPUscout (Sen, Vanecek, Schulz, SC-W 2023; /root/reference/PAPER.md, cited P:line).
 *   - static SASS analysis: pattern checks over the disassembled SASS (§4),
 *     each flagged memory instruction carrying a bounded backward def-use trace;
 *   - warp-stall attribution: PC samples with stall reasons aggregated per PC and
 *     attributed "to the instruction detected by the SASS Analysis engine".
 * Readings of the paper where it is silent are numbered R1..R39 in DESIGN.md §3.
 *
 * Conventions (all entry points):
 *   - Every call returns a gs_status; no exception or abort crosses the ABI. On error the message
 *     is available from gs_last_error(ctx) until the next call on that context.
 *   - A context is bound to one CUDA device and one CUDA stream (given at gs_create). Device work
 *     is enqueued on that stream; calls that return host-visible results synchronise it.
 *   - A context is single-threaded: the caller serialises calls on it.
 *   - "device pointer" arguments must be device memory of the context's device; "host or device"
 *     arguments are classified with cudaPointerGetAttributes. The library never frees caller
 *     memory; buffers it returns (gs_sites) are owned by the context and stay valid until the next
 *     gs_load_sass / gs_detect / gs_destroy.
 */
#ifndef GPUSCOUT_B200_H
#define GPUSCOUT_B200_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  GS_OK = 0,
  GS_E_INVAL = -1,  /* bad argument (null pointer, k_begin > k_end, n_reasons > 32, ...)      */
  GS_E_PARSE = -2,  /* SASS text not understood (message carries the line number)             */
  GS_E_RANGE = -3,  /* size limit exceeded (> 2^31-2 instructions in one context)             */
  GS_E_CUDA = -4,   /* a CUDA runtime call failed (message carries cudaGetErrorString)        */
  GS_E_NOMEM = -5,  /* device or host allocation failed                                        */
  GS_E_STATE = -6   /* call out of order (gs_detect before gs_load_sass, ...)                  */
} gs_status;

typedef struct gs_ctx gs_ctx; /* opaque */

/* Analysis parameters. Zero-initialised fields take the defaults. */
typedef struct {
  uint32_t trace_depth;     /* D: max last-writer steps of a def-use trace (R7). default 64, max 255 */
  uint32_t n_reasons;       /* active stall reasons R (R17, R30). default 19, max 32                 */
  uint32_t shmem_min_arith; /* T_A of the SHMEM rule (R11). default 1                                 */
  uint32_t shmem_min_loads; /* T_L of the SHMEM rule (R11). default 2                                 */
  uint32_t hist_mode;       /* histogram strategy, GS_HIST_*. default GS_HIST_AUTO                    */
  uint32_t hist_counter_bits; /* shared-memory counter width: 0 = auto, 16 (packed pairs) or 32      */
  uint32_t hist_row;        /* bins per histogram row (one row per PC slot): 0 or 32 -> 32 (reason r at
                               column r, the row padded to 32), or n_reasons -> compact rows holding only
                               the active reasons (4*R bytes per slot: less to zero, write and reduce
                               across GPUs). Any other value -> GS_E_INVAL.         */
  uint32_t join_mode;       /* which histogram rows a site is joined with, GS_JOIN_*. default PC     */
} gs_config;

/* Histogram strategies (all exact, they differ only in speed):
 *   GS_HIST_GLOBAL    one L2 atomic per sample (reference strategy);
 *   GS_HIST_PRIVATE   fixed slot ranges per CTA in shared memory (modules of <= 3 tables);
 *   GS_HIST_WINDOW    a shared-memory window that follows the stream (PC-sampling traces, which
 *                     arrive grouped by kernel);
 *   GS_HIST_PARTITION partition by bucket of 2^15 compact bins first (a 16-bit offset per sample),
 *                     then count each bucket in its own table: for streams without locality (random
 *                     order); modules of 2^25 bins (P * R) or more use WINDOW instead;
 *   GS_HIST_AUTO      PRIVATE for small modules, else WINDOW. */
enum { GS_HIST_AUTO = 0, GS_HIST_GLOBAL = 1, GS_HIST_PRIVATE = 2, GS_HIST_WINDOW = 3, GS_HIST_PARTITION = 4 };

/* Join granularity (R18, R33):
 *   GS_JOIN_PC   the site PC's row ("attributed to the instruction detected");
 *   GS_JOIN_LINE the sum of the rows of every instruction of the kernel on the site's source line
 *                (file, line) from nvdisasm -g ("stall reasons ... at the line numbers identified",
 *                P:325-327); a site without line information keeps its PC row.
 *   GS_JOIN_CONSUMER the site PC's row plus the rows of its direct consumers: every instruction j
 *                of the kernel that reads a general-purpose register (pairs expanded) whose last
 *                writer before j is the site instruction (R37; scoreboard stalls are
 *                sampled at the instruction waiting for the data). gs_detect builds the consumer
 *                groups when this mode is configured.
 * Ranked counts[] are the joined row, saturated to 2^32-1; rel and tot are exact. */
enum { GS_JOIN_PC = 0, GS_JOIN_LINE = 1, GS_JOIN_CONSUMER = 2 };

/* Rule ids (paper §4) — also the rank tie-break order. */
enum { GS_VEC = 0, GS_SPILL = 1, GS_SHMEM = 2, GS_GATOM = 3, GS_RO = 4, GS_TEX = 5, GS_CONV = 6 };

/* Trace terminal kinds (R7). */
enum { GS_T_NONE = 0, GS_T_PARAM = 1, GS_T_CONST = 2, GS_T_ENTRY = 3, GS_T_SREG = 4,
       GS_T_MEMORY = 5, GS_T_IMM = 6, GS_T_TRUNC = 7 };

/* One flagged bottleneck site: "type, location, registers, case-specific info".
 * 32 bytes, device-resident, ordered by (kernel, idx, rule).
 *   term_value: PARAM -> offset; CONST -> (bank << 16) | offset; ENTRY -> register id
 *               (GPR n -> n, UR n -> 256 + n); SREG / MEMORY -> kernel-local instruction index.
 *   chain_off : first element in the chain pool; the chain has `depth` kernel-local indices.
 *   a0..a2    : VEC   a0 = distinct offsets | contiguous << 30, a1 = min offset, a2 = max offset
 *               SPILL a0 = data register id, a1 = cause (kernel-local idx; -1 ENTRY; -2 none)
 *               SHMEM a0 = n_loads, a1 = n_arith;   TEX a0 = distinct offsets;   else 0. */
typedef struct {
  uint32_t kernel, idx;
  uint8_t rule, depth, term_kind, loop_depth;
  uint32_t term_value;
  uint32_t chain_off;
  int32_t a0, a1, a2;
} gs_site;

/* Per-kernel counters (R27). */
typedef struct {
  uint32_t n_gatom, n_satom, n_conv, n_vec_already, n_unresolved_stores;
} gs_kernel_stats;

/* One ranked site (host or device output of gs_rank_sites). 168 bytes. */
typedef struct {
  uint32_t kernel, idx, rule, pad;
  uint64_t rel, tot, ktot; /* REL-reason samples and all samples of the joined row, kernel total */
  uint32_t counts[32];     /* the joined histogram row: the site PC row (GS_JOIN_PC), the sum over its  */
                           /* source line (GS_JOIN_LINE) or over it and its consumers (GS_JOIN_CONSUMER);
                              32-bit, saturating (R34)                                               */
} gs_ranked_site;

/* Create a context on `device` that enqueues on `cuda_stream` (a cudaStream_t; NULL = legacy
 * default stream). cfg may be NULL (defaults). */
gs_status gs_create(gs_ctx **out, int device, void *cuda_stream, const gs_config *cfg);
void gs_destroy(gs_ctx *ctx);
const char *gs_last_error(const gs_ctx *ctx);
/* Library build string (arch, version). */
const char *gs_version(void);

/* a-1: parse cuobjdump -sass / nvdisasm [-g] SASS text (host memory, borrowed for the call; `len`
 * bytes, need not be NUL-terminated), pack one 16-byte record per instruction and upload them.
 * Replaces any previously loaded SASS and invalidates sites. Host-synchronous; the upload is
 * enqueued on the context stream. Parse errors -> GS_E_PARSE with the 1-based line number. */
gs_status gs_load_sass(gs_ctx *ctx, const char *text, size_t len, uint32_t *n_kernels, uint64_t *n_instr);

/* Kernel table of the loaded SASS into caller-owned host arrays of capacity `cap` kernels:
 * first_slot[k] = global slot of kernel k's first instruction (slot = first_slot + pc/16),
 * n_instr[k]. Either pointer may be NULL. */
gs_status gs_kernel_table(const gs_ctx *ctx, uint32_t *first_slot, uint32_t *n_instr, size_t cap);
/* Kernel name (NUL-terminated, owned by the context) and source-line table (host array of
 * n_instr entries, -1 where unknown; from nvdisasm "//## File ..., line N"). */
const char *gs_kernel_name(const gs_ctx *ctx, uint32_t k);
gs_status gs_instr_lines(const gs_ctx *ctx, int32_t *lines, size_t cap);

/* a-2..a-7: detection (the paper's dry run) over kernels [k_begin, k_end).
 * Enqueued on the stream; synchronises once at the end to return the site count. With
 * n_sites == NULL it returns without synchronising: the next call that reads the results
 * (gs_sites*, gs_kernel_stats_get, gs_rank_sites*, gs_detect) completes it first, so work enqueued
 * in between (e.g. gs_attribute_samples) follows on the GPU without a host round trip. */
gs_status gs_detect(gs_ctx *ctx, uint32_t k_begin, uint32_t k_end, uint64_t *n_sites);
/* Device pointers to the sites / chain pool of the last gs_detect (owned by the context). */
gs_status gs_sites(const gs_ctx *ctx, const gs_site **d_sites, const uint32_t **d_chain_pool,
                   uint64_t *n_sites, uint64_t *n_chain);
/* Synchronous host copy of the sites (capacity cap_sites) and chain pool (capacity cap_chain) of
 * the last gs_detect; either output may be NULL. */
gs_status gs_sites_host(gs_ctx *ctx, gs_site *sites, size_t cap_sites, uint32_t *chain, size_t cap_chain);
/* Per-kernel counters of the last gs_detect, host array of capacity cap (kernels outside the
 * detected range are zero). */
gs_status gs_kernel_stats_get(const gs_ctx *ctx, gs_kernel_stats *out, size_t cap);

/* a-8: raw samples (device, n x {kernel u32, pc byte offset u32, reason u32}) ->
 * packed words (device, n x u32) word = (first_slot[kernel] + pc/16) * n_reasons + reason (the
 * compact bin index of the sample; requires n_instr * n_reasons < 2^32). Invalid
 * samples (R30) become 0xFFFFFFFF and are counted into *d_n_invalid (device u64, added to).
 * Async. */
gs_status gs_pack_samples(gs_ctx *ctx, const uint32_t *d_raw, uint64_t n, uint32_t *d_words,
                          unsigned long long *d_n_invalid);

/* a-9: H[slot*row + reason] += 1 for every valid packed word w = slot * n_reasons +
 * reason (valid iff w < n_instr * n_reasons; row = gs_config.hist_row, 32 by default); others are
 * counted into *d_n_invalid (device u64, added to). `samples` may be host
 * (pinned or pageable; streamed in chunks with copies overlapped) or device memory. d_hist is a
 * caller-owned device int32 array of n_instr*row bins, zeroed first unless accumulate != 0.
 * Async for device input; host input returns after the last chunk is consumed. */
gs_status gs_attribute_samples(gs_ctx *ctx, const uint32_t *samples, uint64_t n, int32_t *d_hist,
                               unsigned long long *d_n_invalid, int accumulate);

/* a-9 for PRE-AGGREGATED PC-sampling data (CUPTI's CUpti_PCSamplingPCData gives, per PC, a sample
 * count per stall reason): d_recs (device) holds n records of four
 * uint32 {kernel, pc byte offset, reason, count}; H[slot*row + reason] += count for every valid
 * record (validity as gs_pack_samples, R30), and *d_n_invalid (device u64) += count of every
 * invalid one, so that sum(H) + n_invalid = sum(count). d_hist (device, n_instr*row int32) is
 * zeroed first unless accumulate != 0; bins must stay below 2^31. Async. */
gs_status gs_attribute_counts(gs_ctx *ctx, const uint32_t *d_recs, uint64_t n, int32_t *d_hist,
                              unsigned long long *d_n_invalid, int accumulate);

/* CUPTI PC-sampling ingest (§2.2; R39).
 * gs_cupti_stall_reasons: the stall-reason table of cuptiPCSamplingGetStallReasons — n CUPTI
 * indices and their names ("smsp__pcsamp_warps_issue_stalled_<reason>[_not_issued]", host strings,
 * borrowed for the call). A name maps to one of the 19 ncu reasons (R17); "_not_issued" counters are
 * a subset of the same samples and are skipped; other names are unknown (invalid). Kept until the
 * next call. */
gs_status gs_cupti_stall_reasons(gs_ctx *ctx, size_t n, const uint32_t *index, const char *const *names);
/* gs_attribute_cupti: pc_data = CUpti_PCSamplingPCData[n_pcs] (cupti_pcsampling.h, 64-byte records,
 * HOST memory as CUPTI returns it: functionName and stallReason are host pointers). Every
 * (record, stall reason) adds its samples to H[slot*row + reason] with kernel = the loaded kernel
 * named functionName, slot = first_slot + pcOffset/16; records of another cubin (cubin_crc != 0 and
 * record crc different), an unknown function or reason, or an invalid pc (R30) add their samples to
 * *d_n_invalid (device u64); skipped (_not_issued) samples are counted into *n_skipped (host, may be
 * NULL); *n_records (host, may be NULL) = the flattened (record, reason) entries. d_hist as
 * gs_attribute_counts (zeroed unless accumulate). The flattening runs on host threads into pinned
 * memory; returns when the staging copy is done (the scatter-add is async). */
gs_status gs_attribute_cupti(gs_ctx *ctx, const void *pc_data, size_t n_pcs, uint64_t cubin_crc, int32_t *d_hist,
                             unsigned long long *d_n_invalid, int accumulate, unsigned long long *n_skipped,
                             unsigned long long *n_records);

/* a-11, a-12 (R20): join the (already all-reduced) histogram onto the sites of the
 * last gs_detect (rows per gs_config.join_mode) and rank them by (rel desc, tot desc, kernel, idx,
 * rule). Writes the first
 * min(k, n_sites) rows to `out` (host or device; k = UINT64_MAX -> all) and the row count to
 * *n_out. Synchronises the stream. */
gs_status gs_rank_sites(gs_ctx *ctx, const int32_t *d_hist, uint64_t k, gs_ranked_site *out,
                        uint64_t *n_out);
/* Same as gs_rank_sites against a histogram SLICE: d_hist (device) holds the rows of slots
 * [slot_begin, slot_end) only (row width gs_config.hist_row), e.g. this rank's part after a
 * reduce-scatter of the histogram by the kernel-aligned slot ranges of the detection shards
 * (SURVEY §8e, §8f row 1). The slice must cover every slot of the kernels of the last gs_detect,
 * else GS_E_RANGE. ktot is computed for those kernels only. gs_rank_sites(ctx, h, ...) ==
 * gs_rank_sites_slice(ctx, h, 0, n_instr, ...). Synchronises the stream. */
gs_status gs_rank_sites_slice(gs_ctx *ctx, const int32_t *d_hist, uint64_t slot_begin, uint64_t slot_end,
                              uint64_t k, gs_ranked_site *out, uint64_t *n_out);

/* Register pressure ("the number of additional registers needed by each SASS
 * instruction"; also P:452): for every instruction of
 * kernels [k_begin, k_end), the number of general-purpose registers (R0..R254) live at it,
 * |live_in ∪ defs| by backward dataflow over the kernel's control-flow graph (R36; equal
 * to nvdisasm's life-range "GPR #" column). d_live is a caller-owned DEVICE array indexed by global
 * slot (n_instr entries); slots outside the range are left untouched. The additional registers of
 * instruction i are d_live[i] - d_live[i-1] (the first instruction of a kernel: d_live[i]).
 * Enqueued on the stream; synchronises once (basic-block count). */
gs_status gs_register_pressure(gs_ctx *ctx, uint32_t k_begin, uint32_t k_end, uint16_t *d_live);

/* Number of CUDA kernels this library has launched in the process so far (its own kernels plus
 * the CUB radix-sort kernels of gs_rank_sites). Lets a harness count launches in a timed region. */
uint64_t gs_launch_count(void);

/* Histogram strategy actually used by the last gs_attribute_samples (GS_HIST_*). */
int gs_last_hist_mode(const gs_ctx *ctx);

/* GPU time in milliseconds of the device work of the last gs_attribute_samples call with device
 * input (histogram zeroing, planning and counting kernels): two CUDA events recorded on the
 * context's stream, the first after the call's host-side preparation and before its first
 * enqueue, the second after its last enqueue, so host launch gaps before the pass are excluded.
 * Waits for the second event. GS_E_STATE if there was no such call (or the last one had host
 * input). A measurement aid for harnesses (bench.py's roofline); computes nothing. */
gs_status gs_last_attribute_ms(gs_ctx *ctx, float *ms);

#ifdef __cplusplus
}
#endif
#endif
