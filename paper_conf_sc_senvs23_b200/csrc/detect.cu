// detect.cu — SASS detection on the GPU (SURVEY §8a rows a-2 .. a-7; paper §4).
//
// Data layout: records (16 B each, one uint4 per lane) are processed in windows of c->win
// instructions that never cross a kernel. One warp owns one window.
//
//   k_summary  per window: last writer of every register inside the window (R5), loop events of
//              backward branches (R13), per-kernel opcode counters.
//   k_carry    per kernel: turns window summaries into carry-in tables (segmented prefix), loop
//              depth carry-in per window.
//   k_resolve  per window: reaching definitions RD(i, r) for the pointer operand of
//              every instruction and for the address base / spilled register of every
//              candidate; loop depth; n_arith of global loads.
//              Within a 32-instruction chunk the last earlier writer of a register comes from a
//              warp-wide writer bitmask in shared memory (atomicOr + clz), across chunks and
//              windows from the carried table.
//   k_trace    per candidate: bounded backward def-use trace (R7) by pointer chasing
//              through the per-instruction pointer-operand RD; store roots (R8); key-group
//              statistics of global loads (R3).
//   k_rules    per candidate: the seven rules -> flag mask and site count.
//   scans      site offsets and chain-pool offsets.
//   k_write    per candidate: gs_site records in (kernel, idx, rule) order + chains.
#include <cuda_runtime.h>

#include <climits>
#include <cstring>
#include <cstdio>

#include "ctx.h"

namespace gs {
namespace {

constexpr uint64_t kEmpty = ~0ull;
constexpr int kWarps = 8;  // warps (windows) per CTA in the window kernels
#ifndef GS_RES_MINB
#define GS_RES_MINB 5  // resident CTAs per SM the window kernels are compiled for (register budget)
#endif
#ifndef GS_SUM_MINB
#define GS_SUM_MINB 5
#endif

__device__ __forceinline__ Rec ld_rec(const Rec* r, uint64_t i) {
  uint4 v = __ldg(reinterpret_cast<const uint4*>(r) + i);
  Rec o;
  o.w0 = v.x; o.w1 = v.y; o.w2 = v.z; o.w3 = (int32_t)v.w;
  return o;
}
// a record written earlier by the same kernel (not through the read-only path)
__device__ __forceinline__ Rec ld_rec_rw(const Rec* r, uint64_t i) {
  const uint4 v = reinterpret_cast<const uint4*>(r)[i];
  Rec o;
  o.w0 = v.x; o.w1 = v.y; o.w2 = v.z; o.w3 = (int32_t)v.w;
  return o;
}
__device__ __forceinline__ uint32_t reg_cap(uint32_t dst) { return dst < 256 ? 254u : 318u; }
// The opcode-class table in shared memory: op_class() is a switch that compiles to a branch tree,
// which a warp of mixed opcodes walks divergently for every record; one LDS replaces it. The table
// is evaluated at compile time and copied in with one load per entry (evaluating the switch in
// every CTA's prologue was 13% of k_trace's instructions).
struct ClsTable {
  uint16_t v[OP_COUNT];
};
constexpr ClsTable make_cls_table() {
  ClsTable t{};
  for (uint32_t i = 0; i < OP_COUNT; i++) t.v[i] = (uint16_t)op_class(i);
  return t;
}
__device__ const ClsTable g_cls = make_cls_table();
__device__ __forceinline__ void opcls_init(uint16_t* t) {
  for (uint32_t i = threadIdx.x; i < OP_COUNT; i += blockDim.x) t[i] = __ldg(&g_cls.v[i]);
}

// f(q < nq, base + q) for the first four registers of a destination (unrolled: no divergent loop
// for the usual widths 1, 2, 4; k_summary 262 -> 235 us on C3), a loop for wider destinations
template <typename F>
__device__ __forceinline__ void for_regs(uint32_t base, uint32_t nq, F f) {
  f(nq > 0, base);
  f(nq > 1, base + 1);
  f(nq > 2, base + 2);
  f(nq > 3, base + 3);
  for (uint32_t q = 4; q < nq; q++) f(true, base + q);
}

__device__ __forceinline__ uint32_t hash64(unsigned long long k) {
  k ^= k >> 33; k *= 0xff51afd7ed558ccdull; k ^= k >> 33; k *= 0xc4ceb9fe1a85ec53ull; k ^= k >> 33;
  return (uint32_t)k;
}
// Open addressing inside one kernel's region [base, base + mask + 1) of a table whose entries are
// `stride` 8-byte words apart (the key is the entry's first word); returns the region-relative slot.
template <int kStride>
__device__ uint32_t hinsert(unsigned long long* tab, uint32_t mask, unsigned long long k) {
  uint32_t s = hash64(k) & mask;
  for (;;) {
    unsigned long long prev = atomicCAS(tab + (uint64_t)s * kStride, kEmpty, k);
    if (prev == kEmpty || prev == k) return s;
    s = (s + 1) & mask;
  }
}
__device__ bool hcontains(const unsigned long long* keys, uint32_t mask, unsigned long long k) {
  uint32_t s = hash64(k) & mask;
  for (;;) {
    unsigned long long v = keys[s];
    if (v == k) return true;
    if (v == kEmpty) return false;
    s = (s + 1) & mask;
  }
}
__device__ __forceinline__ unsigned long long root_key(uint32_t kernel, uint32_t tk, uint32_t tv) {
  return ((unsigned long long)kernel << 36) | ((unsigned long long)tk << 32) | tv;
}
// key of a global load's group (R3): (base register, RD(i, base)); ENTRY / no-base keys are per kernel
__device__ __forceinline__ unsigned long long group_key(uint32_t base, uint32_t base_rd, uint32_t kernel) {
  if (!reg_live(base)) return (2ull << 62) | ((unsigned long long)kernel << 10) | (base & 1023u);
  if (base_rd == 0) return (1ull << 62) | ((unsigned long long)kernel << 10) | base;
  return ((unsigned long long)base_rd << 10) | base;
}

// Programmatic dependent launch between consecutive detection kernels: a primary lets its
// dependent grid launch once all its CTAs are running (pdl_trigger); the dependent's CTAs fill the
// SMs the primary frees and wait (pdl_wait) for its completion before touching its outputs.
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

// ------------------------------------------------------------------------------------------ A
__global__ void __launch_bounds__(kWarps * 32, GS_SUM_MINB) k_summary(const Rec* __restrict__ rec, const WDesc* __restrict__ wd,
                                                         const KDesc* __restrict__ kd, uint32_t w0, uint32_t nw,
                                                         uint32_t* __restrict__ tab, int32_t* ldiff, int32_t* wsum,
                                                         uint32_t* wev, uint32_t* narith, gs_kernel_stats* kst,
                                                         uint32_t win) {
  __shared__ uint32_t last[kWarps][kNumRegs];
  __shared__ uint16_t s_cls[OP_COUNT];
  pdl_trigger();
  opcls_init(s_cls);
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t w = w0 + blockIdx.x * kWarps + warp;
  if (w >= w0 + nw) return;
  for (int r = lane; r < kNumRegs; r += 32) last[warp][r] = 0;
  __syncwarp();
  const WDesc W = wd[w];
  const KDesc K = kd[W.kernel];
  uint32_t n_gatom = 0, n_satom = 0, n_conv = 0, n_vec = 0;
  constexpr int kAhead = 4;  // chunks whose records are loaded together (no cross-chunk dependency)
  for (uint32_t b0 = 0; b0 < W.len; b0 += 32 * kAhead) {
    Rec rr[kAhead];
#pragma unroll
    for (int u = 0; u < kAhead; u++) {
      const uint32_t i = b0 + 32 * u + lane;
      rr[u] = i < W.len ? ld_rec(rec, (uint64_t)W.start + i) : Rec{0, 0, 0, 0};
    }
#pragma unroll
    for (int u = 0; u < kAhead; u++) {
    const uint32_t i = b0 + 32 * u + lane;
    const bool valid = i < W.len;
    const uint64_t g = (uint64_t)W.start + i;
    const Rec r = rr[u];
    const uint32_t op = r_op(r), cls = s_cls[op], dst = r_dst(r), dw = r_dstw(r), dst2 = r_dst2(r);
    if (valid && dw && reg_live(dst)) {
      const uint32_t v = (uint32_t)((g + 1) << 1) | (op == OP_LDG ? 1u : 0u);
      const uint32_t nq = min(dw, reg_cap(dst) + 1 - dst);
      for_regs(dst, nq, [&](bool p, uint32_t x) { if (p) atomicMax(&last[warp][x], v); });
      if (reg_live(dst2)) {  // second quad of a 256-bit load (R38a)
        const uint32_t nq2 = min(dw, reg_cap(dst2) + 1 - dst2);
        for_regs(dst2, nq2, [&](bool p, uint32_t x) { if (p) atomicMax(&last[warp][x], v); });
      }
    }
    if (valid && op == OP_LDG) narith[g] = 0;
    if (valid && op == OP_BRA && (r_flags(r) & F_BRA_OK)) {
      const uint32_t t = (uint32_t)r_imm(r);           // loop [t, b] in kernel-local indices
      atomicAdd(ldiff + K.first + t, 1);
      atomicAdd(wsum + K.win0 + t / win, 1);
      atomicAdd(wev + K.win0 + t / win, 1u);
      const uint32_t b1 = (uint32_t)(g - K.first) + 1;
      if (b1 < K.n) {
        atomicAdd(ldiff + K.first + b1, -1);
        atomicAdd(wsum + K.win0 + b1 / win, -1);
        atomicAdd(wev + K.win0 + b1 / win, 1u);
      }
    }
    if (valid) {
      n_gatom += (cls & C_GATOM) ? 1 : 0;
      n_satom += (cls & C_SATOM) ? 1 : 0;
      n_conv += (cls & C_CONV) ? 1 : 0;
      n_vec += (op == OP_LDG && (r_flags(r) & F_HASMEM) && (r_aw(r) == AW_64 || r_aw(r) == AW_128 || r_aw(r) == AW_256))
                   ? 1 : 0;  // "already vectorised" (R38a)
    }
    }
  }
  for (int o = 16; o; o >>= 1) {
    n_gatom += __shfl_xor_sync(0xffffffffu, n_gatom, o);
    n_satom += __shfl_xor_sync(0xffffffffu, n_satom, o);
    n_conv += __shfl_xor_sync(0xffffffffu, n_conv, o);
    n_vec += __shfl_xor_sync(0xffffffffu, n_vec, o);
  }
  if (lane == 0) {
    if (n_gatom) atomicAdd(&kst[W.kernel].n_gatom, n_gatom);
    if (n_satom) atomicAdd(&kst[W.kernel].n_satom, n_satom);
    if (n_conv) atomicAdd(&kst[W.kernel].n_conv, n_conv);
    if (n_vec) atomicAdd(&kst[W.kernel].n_vec_already, n_vec);
  }
  __syncwarp();
  for (int r = lane; r < kNumRegs; r += 32) tab[(uint64_t)w * kNumRegs + r] = last[warp][r];
}

// ------------------------------------------------------------------------------------------ B
__global__ void k_carry(const KDesc* __restrict__ kd, uint32_t kb, uint32_t ke, uint32_t* tab,
                        const int32_t* __restrict__ wsum, int32_t* wloop, uint32_t win) {
  pdl_wait();
  pdl_trigger();
  const uint32_t k = kb + blockIdx.x;
  if (k >= ke) return;
  const KDesc K = kd[k];
  const uint32_t nwk = (K.n + win - 1) / win;
  for (int r = threadIdx.x; r < kNumRegs; r += blockDim.x) {
    {
      uint32_t state = 0;
      constexpr uint32_t kB = 8;  // window summaries loaded per batch
      for (uint32_t j0 = 0; j0 < nwk; j0 += kB) {
        uint32_t v[kB];
#pragma unroll
        for (uint32_t u = 0; u < kB; u++)
          v[u] = j0 + u < nwk ? tab[(uint64_t)(K.win0 + j0 + u) * kNumRegs + r] : 0u;
#pragma unroll
        for (uint32_t u = 0; u < kB; u++) {
          if (j0 + u < nwk) tab[(uint64_t)(K.win0 + j0 + u) * kNumRegs + r] = state;
          if (v[u]) state = v[u];
        }
      }
    }
  }
  if (threadIdx.x >= kNumRegs && threadIdx.x < kNumRegs + 32) {  // loop-depth carry-in: warp scan
    const int lane = threadIdx.x & 31;
    int32_t acc = 0;
    for (uint32_t j0 = 0; j0 < nwk; j0 += 32) {
      const uint32_t j = j0 + lane;
      int32_t x = j < nwk ? wsum[K.win0 + j] : 0;
      int32_t inc = x;
      for (int o = 1; o < 32; o <<= 1) {
        const int32_t y = __shfl_up_sync(0xffffffffu, inc, o);
        if (lane >= o) inc += y;
      }
      if (j < nwk) wloop[K.win0 + j] = acc + inc - x;
      acc += __shfl_sync(0xffffffffu, inc, 31);
    }
  }
}

// ------------------------------------------------------------------------------------------ D0
struct TraceOut {
  uint32_t tk, tv, depth, cont;
};
constexpr uint32_t kTCont = 0xFEu;
constexpr uint32_t kChain4 = 4;  // chain elements kept per candidate  // internal term kind: the trace continues before `lo` (resumed later)

// Bounded backward trace (R7) from the state (register r, its RD value v, steps taken):
// each step j = v - 1 is emitted (kernel-local) and classified; a step that would read an instruction
// below `lo` (an earlier window, whose RDs another warp may still be resolving) stops with
// tk = kTCont, tv = r, cont = v, to be resumed from exactly that state.
template <typename Emit>
__device__ TraceOut chase_from(const Rec* __restrict__ rec, const uint32_t* ptrrd, const KDesc& K, uint32_t r,
                               uint32_t v, uint32_t depth, uint32_t D, uint64_t lo,
                               const uint16_t* __restrict__ cls_tab, Emit emit) {
  TraceOut o{GS_T_IMM, 0, 0, 0};
  for (;;) {
    if (depth == D) { o.tk = GS_T_TRUNC; break; }
    if (v == 0) { o.tk = GS_T_ENTRY; o.tv = r; break; }
    const uint32_t j = v - 1;
    if (j < lo) { o.tk = kTCont; o.tv = r; o.cont = v; break; }
    depth++;
    emit(j - K.first);
    const Rec rj = ld_rec(rec, j);
    const uint32_t cj = cls_tab[r_op(rj)];
    if (cj & C_CONSTLOAD) {
      const int32_t off = r_imm(rj) + 4 * (int32_t)(r - r_dst(rj));
      const uint32_t bank = r_cbank(rj);
      if (bank == 0 && off >= (int32_t)kd_param_base(K)) { o.tk = GS_T_PARAM; o.tv = (uint32_t)off; }
      else { o.tk = GS_T_CONST; o.tv = (bank << 16) | ((uint32_t)off & 0xffffu); }
      break;
    }
    if (cj & C_SREG) { o.tk = GS_T_SREG; o.tv = j - K.first; break; }
    if (cj & C_MEMLOAD) { o.tk = GS_T_MEMORY; o.tv = j - K.first; break; }
    const uint32_t pk = r_pk(rj);
    if (pk == PK_CONST) {
      const int32_t off = r_imm(rj);
      const uint32_t bank = r_cbank(rj);
      if (bank == 0 && off >= (int32_t)kd_param_base(K)) { o.tk = GS_T_PARAM; o.tv = (uint32_t)off; }
      else { o.tk = GS_T_CONST; o.tv = (bank << 16) | ((uint32_t)off & 0xffffu); }
      break;
    }
    if (pk != PK_REG) { o.tk = GS_T_IMM; break; }
    r = r_ptr(rj);
    v = ptrrd[j];
  }
  o.depth = depth;
  return o;
}
// the whole trace of a candidate with address base `base` and RD(base) = base_rd
template <typename Emit>
__device__ TraceOut chase(const Rec* __restrict__ rec, const uint32_t* ptrrd, const KDesc& K, uint32_t base,
                          uint32_t base_rd, uint32_t D, const uint16_t* __restrict__ cls_tab, Emit emit) {
  if (!reg_live(base) || base_rd == 0xffffffffu) return TraceOut{GS_T_IMM, 0, 0, 0};
  return chase_from(rec, ptrrd, K, base, base_rd, 0, D, 0, cls_tab, emit);
}

// ------------------------------------------------------------------------------------------ C
// One warp per window. Per 32-instruction chunk: (1) every lane marks the registers its instruction
// writes in the chunk's writer bitmasks M; (2) lookups RD(i, reg) = the highest earlier lane of the
// chunk whose bit is set in M[reg], else the carried table T[reg]; (3) T[reg] = max(T[reg], v) (v
// grows with the instruction index, so the chunk's last writer wins) and M is cleared. n_arith of
// loads defined inside the window is counted in shared memory (16-bit halves) and added to the
// global array once per window. At the end of the window the warp traces the window's candidates
// while their steps stay inside the window (the RDs of earlier windows belong to other warps);
// k_trace resumes the others.
constexpr uint32_t kNarWords = kWinBig / 2;  // 16-bit n_arith counters per window instruction
__global__ void __launch_bounds__(kWarps * 32, GS_RES_MINB) k_resolve(const Rec* __restrict__ rec, const WDesc* __restrict__ wd,
                                                         const KDesc* __restrict__ kd, uint32_t w0, uint32_t nw,
                                                         const uint32_t* __restrict__ tab, int32_t* ldiff,
                                                         const int32_t* __restrict__ wloop,
                                                         const uint32_t* __restrict__ wev,
                                                         const uint32_t* __restrict__ cbase, uint64_t c0,
                                                         uint32_t* ptrrd, uint32_t* narith, CandArrays ca, uint32_t D) {
  __shared__ uint2 mtS[kWarps][kNumRegs];  // per register: {writer lanes of the chunk M, carried table T}
  __shared__ uint32_t nar[kWarps][kNarWords];
  __shared__ uint16_t s_cls[OP_COUNT];
  opcls_init(s_cls);
  pdl_wait();
  __syncthreads();
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t w = w0 + blockIdx.x * kWarps + warp;
  if (w >= w0 + nw) return;
  const WDesc W = wd[w];
  {  // the window's carried table: all ten loads of a lane in flight before the first store
    static_assert(kNumRegs % 32 == 0, "registers per lane");
    uint32_t tv[kNumRegs / 32];
#pragma unroll
    for (int u = 0; u < kNumRegs / 32; u++) tv[u] = __ldg(tab + (uint64_t)w * kNumRegs + lane + 32 * u);
#pragma unroll
    for (int u = 0; u < kNumRegs / 32; u++) mtS[warp][lane + 32 * u] = make_uint2(0u, tv[u]);
    for (uint32_t q = lane; q < (W.len + 1) / 2; q += 32) nar[warp][q] = 0;
  }
  __syncwarp();
  int32_t lcarry = wloop[w];
  const bool has_ev = wev[w] != 0;
  const uint64_t cb0 = (uint64_t)cbase[w] - c0;
  uint64_t cb = cb0;
  const uint32_t lt = (1u << lane) - 1u;
  uint2* MT = mtS[warp];
  uint32_t* NA = nar[warp];
  // records (and loop events) of the next two chunks load while a chunk resolves
  Rec rn1 = lane < W.len ? ld_rec(rec, (uint64_t)W.start + lane) : Rec{0, 0, 0, 0};
  Rec rn2 = lane + 32 < W.len ? ld_rec(rec, (uint64_t)W.start + lane + 32) : Rec{0, 0, 0, 0};
  int32_t dn1 = has_ev && lane < W.len ? ldiff[(uint64_t)W.start + lane] : 0;
  int32_t dn2 = has_ev && lane + 32 < W.len ? ldiff[(uint64_t)W.start + lane + 32] : 0;
  for (uint32_t b = 0; b < W.len; b += 32) {
    const uint32_t i = b + lane;
    const bool valid = i < W.len;
    const uint32_t g = W.start + i, gbase = W.start + b;  // slots < 2^31: RD values fit 32 bits
    const Rec r = rn1;
    const int32_t dcur = dn1;
    rn1 = rn2;
    dn1 = dn2;
    rn2 = i + 64 < W.len ? ld_rec(rec, g + 64) : Rec{0, 0, 0, 0};
    if (has_ev) dn2 = i + 64 < W.len ? ldiff[g + 64] : 0;
    const uint32_t op = r_op(r), cls = s_cls[op], dst = r_dst(r), fl = r_flags(r);
    const bool writes = valid && r_dstw(r) && reg_live(dst);
    const uint32_t nq = writes ? min(r_dstw(r), reg_cap(dst) + 1 - dst) : 0u;
    const uint32_t dst2 = writes ? r_dst2(r) : (uint32_t)kRegNone;  // second quad (R38a)
    const uint32_t nq2 = reg_live(dst2) ? min(r_dstw(r), reg_cap(dst2) + 1 - dst2) : 0u;
    // (predicated per register: unconditional atomics with idle lanes on one dummy entry were
    // measured 20% slower on C3, same-address conflicts)
    const auto mark = [&](bool p, uint32_t x) { if (p) atomicOr(&MT[x].x, 1u << lane); };
    for_regs(dst, nq, mark);
    if (nq2) for_regs(dst2, nq2, mark);
    const uint32_t ldgmask = __ballot_sync(0xffffffffu, valid && op == OP_LDG);
    __syncwarp();
    // loop depth: inclusive prefix of the event differences (R13); a window without loop events
    // (warp-uniform) keeps its carried depth
    int32_t depth = lcarry;
    if (has_ev) {
      int32_t pre = dcur;
      if (pre) ldiff[g] = 0;  // keep the difference array zero for the next call
      for (int o = 1; o < 32; o <<= 1) {
        const int32_t x = __shfl_up_sync(0xffffffffu, pre, o);
        if (lane >= o) pre += x;
      }
      depth = lcarry + pre;
      lcarry += __shfl_sync(0xffffffffu, pre, 31);
    }
    // RD value: ((def + 1) << 1) | def_is_global_load, or 0 for ENTRY (a flat, predicated form of
    // the lookups measured slower: 962 vs 915 us on C3, more instructions)
    auto RD = [&](uint32_t reg) -> uint32_t {
      const uint2 mt = MT[reg];
      const uint32_t m = mt.x & lt;
      const uint32_t j = 31u - __clz(m);
      return m ? ((gbase + j + 1) << 1) | ((ldgmask >> j) & 1u) : mt.y;
    };
    if (valid && r_pk(r) == PK_REG) ptrrd[g] = RD(r_ptr(r)) >> 1;
    const bool iscand = valid && (cls & (C_TRACED | C_CONV));
    const uint32_t cmask = __ballot_sync(0xffffffffu, iscand);
    if (iscand) {
      const uint64_t c = cb + __popc(cmask & lt);
      ca.idx[c] = g;
      ca.kernel[c] = W.kernel;
      reinterpret_cast<uint4*>(ca.rec)[c] = make_uint4(r.w0, r.w1, r.w2, (uint32_t)r.w3);
      const uint32_t base = r_s0(r);
      ca.base_rd[c] = ((fl & F_HASMEM) && reg_live(base)) ? (RD(base) >> 1) : 0xffffffffu;
      const uint32_t data = r_s1(r);
      ca.data_rd[c] = (op == OP_STL && reg_live(data)) ? (RD(data) >> 1) : 0xffffffffu;
      ca.ld[c] = (uint8_t)(depth > 255 ? 255 : (depth < 0 ? 0 : depth));
    }
    cb += __popc(cmask);
    if (valid && (cls & C_ARITH)) {  // n_arith (R29): count each defining load once
      const uint32_t src[4] = {r_s0(r), r_s1(r), r_s2(r), r_s3(r)};
      uint32_t d[4];
#pragma unroll
      for (int q = 0; q < 4; q++) {
        const uint32_t v = reg_live(src[q]) ? RD(src[q]) : 0u;
        d[q] = (v & 1u) ? (v >> 1) - 1u : ~0u;  // the defining load, ~0u if none
      }
#pragma unroll
      for (int q = 0; q < 4; q++) {
        bool dup = d[q] == ~0u;
#pragma unroll
        for (int t = 0; t < q; t++) dup |= d[t] == d[q];
        if (dup) continue;
        const uint32_t off = d[q] - W.start;  // loads of this window: shared counters
        if (off < W.len) atomicAdd(NA + (off >> 1), 1u << ((off & 1u) << 4));
        else atomicAdd(narith + d[q], 1u);
      }
    }
    __syncwarp();
    {  // the chunk's last writer of a register (the highest lane of its mask) sets T and clears M;
       // only that lane writes the entry, so no atomic is needed
      const uint32_t v = ((g + 1) << 1) | (op == OP_LDG ? 1u : 0u);
      const auto last = [&](bool p, uint32_t x) {
        if (p && (MT[x].x >> lane) == 1u) MT[x] = make_uint2(0u, v);
      };
      for_regs(dst, nq, last);
      if (nq2) for_regs(dst2, nq2, last);
    }
    __syncwarp();
  }
  // n_arith of the window's loads (k_summary zeroed their entries; later windows add theirs)
  for (uint32_t i = lane; i < W.len; i += 32) {
    const uint32_t n = (NA[i >> 1] >> ((i & 1u) << 4)) & 0xffffu;
    if (n) atomicAdd(narith + W.start + i, n);
  }
  // in-window traces of the window's candidates (ptrrd of the window is complete and visible to
  // the warp after the __syncwarp above)
  const KDesc K = kd[W.kernel];
  for (uint64_t c = cb0 + lane; c < cb; c += 32) {
    const Rec ri = ld_rec_rw(ca.rec, c);
    const uint32_t cls = s_cls[r_op(ri)];
    TraceOut tr{GS_T_NONE, 0, 0, 0};
    uint32_t e0 = 0, e1 = 0, e2 = 0, e3 = 0, n = 0;  // the first chain elements (k_write copies them)
    if ((cls & C_TRACED) && (r_flags(ri) & F_HASMEM)) {
      const uint32_t base = r_s0(ri), brd = ca.base_rd[c];
      tr = reg_live(base) && brd != 0xffffffffu
               ? chase_from(rec, ptrrd, K, base, brd, 0, D, W.start, s_cls,
                            [&](uint32_t j) {
                              e0 = n == 0 ? j : e0;
                              e1 = n == 1 ? j : e1;
                              e2 = n == 2 ? j : e2;
                              e3 = n == 3 ? j : e3;
                              n++;
                            })
               : TraceOut{GS_T_IMM, 0, 0, 0};
      reinterpret_cast<uint4*>(ca.chain4)[c] = make_uint4(e0, e1, e2, e3);
    }
    ca.tk[c] = (uint8_t)tr.tk;
    ca.tv[c] = tr.tv;
    ca.depth[c] = (uint8_t)tr.depth;
    ca.cont[c] = tr.cont;
  }
}

// ------------------------------------------------------------------------------------------ C'
// Consumer join (GS_JOIN_CONSUMER, reading R37; [probe 9]: scoreboard stalls are sampled at the
// instruction that waits for the data). Per window (one warp), the same reaching-definition
// machinery as k_resolve: for every GPR use q of instruction j (the packer's use lists, pairs
// expanded as in R36) cdef[q] = RD(j, reg) (~0u for ENTRY or when j already reads another
// register of the same definition), and ccnt[def] += 1.
__global__ void __launch_bounds__(kWarps * 32) k_consumers(const Rec* __restrict__ rec, const WDesc* __restrict__ wd,
                                                           uint32_t w0, uint32_t nw, const uint32_t* __restrict__ tab,
                                                           const uint32_t* __restrict__ use_off,
                                                           const uint8_t* __restrict__ use_reg, uint32_t* cdef,
                                                           uint32_t* ccnt) {
  __shared__ uint32_t tabS[kWarps][256];  // GPR entries of the carried last-writer table
  __shared__ uint32_t cm[kWarps][256];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t w = w0 + blockIdx.x * kWarps + warp;
  if (w >= w0 + nw) return;
  {
    uint32_t tv[8];
#pragma unroll
    for (int u = 0; u < 8; u++) tv[u] = __ldg(tab + (uint64_t)w * kNumRegs + lane + 32 * u);
#pragma unroll
    for (int u = 0; u < 8; u++) {
      tabS[warp][lane + 32 * u] = tv[u];
      cm[warp][lane + 32 * u] = 0;
    }
  }
  __syncwarp();
  const WDesc W = wd[w];
  const uint32_t lt = (1u << lane) - 1u;
  const uint32_t gt = ~((2u << lane) - 1u);
  uint32_t* T = tabS[warp];
  uint32_t* M = cm[warp];
  for (uint32_t b = 0; b < W.len; b += 32) {
    const uint32_t i = b + lane;
    const bool valid = i < W.len;
    const uint64_t g = (uint64_t)W.start + i;
    const uint64_t gbase = (uint64_t)W.start + b;
    const Rec r = valid ? ld_rec(rec, g) : Rec{0, 0, 0, 0};
    const uint32_t dst = r_dst(r), dw = r_dstw(r);
    const bool writes = valid && dw && dst < 255;  // GPR definitions only
    const uint32_t dst2 = writes ? r_dst2(r) : (uint32_t)kRegNone;  // second quad (R38a)
    const bool writes2 = dst2 < 255;
    if (writes)
      for (uint32_t q = 0; q < dw && dst + q < 255; q++) atomicOr(&M[dst + q], 1u << lane);
    if (writes2)
      for (uint32_t q = 0; q < dw && dst2 + q < 255; q++) atomicOr(&M[dst2 + q], 1u << lane);
    __syncwarp();
    if (valid) {
      const uint32_t q0 = use_off[g], q1 = use_off[g + 1];
      for (uint32_t q = q0; q < q1; q++) {
        const uint32_t reg = use_reg[q];
        const uint32_t m = M[reg] & lt;
        const uint32_t v = m ? (uint32_t)((gbase + (31u - __clz(m)) + 1) << 1) : T[reg];
        uint32_t d = v ? (v >> 1) - 1u : ~0u;
        for (uint32_t p = q0; p < q && d != ~0u; p++)
          if (cdef[p] == d) d = ~0u;  // j counts once per definition
        cdef[q] = d;
        if (d != ~0u) atomicAdd(ccnt + d, 1u);
      }
    }
    __syncwarp();
    if (writes) {
      const uint32_t v = (uint32_t)((g + 1) << 1);
      for (uint32_t q = 0; q < dw && dst + q < 255; q++)
        if ((M[dst + q] & gt) == 0) T[dst + q] = v;
      if (writes2)
        for (uint32_t q = 0; q < dw && dst2 + q < 255; q++)
          if ((M[dst2 + q] & gt) == 0) T[dst2 + q] = v;
    }
    __syncwarp();
    if (writes)
      for (uint32_t q = 0; q < dw && dst + q < 255; q++) M[dst + q] = 0;
    if (writes2)
      for (uint32_t q = 0; q < dw && dst2 + q < 255; q++) M[dst2 + q] = 0;
    __syncwarp();
  }
}

// slots [s0, s0 + n): 1 (the slot's own row) before the consumers are counted; ccnt[s0 + n] = 0
__global__ void k_cons_init(uint32_t* ccnt, uint64_t s0, uint64_t n) {
  const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (i <= n) ccnt[s0 + i] = i < n ? 1u : 0u;
}

// group of slot s = {s, its consumers}: gslot[goff[s]] = s, consumers after it (any order)
__global__ void k_cons_fill(uint64_t s0, uint64_t n, const uint32_t* __restrict__ use_off,
                            const uint32_t* __restrict__ cdef, const uint32_t* __restrict__ goff, uint32_t* ccnt,
                            uint32_t* gslot) {
  const uint64_t s = s0 + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (s >= s0 + n) return;
  gslot[goff[s]] = (uint32_t)s;
  for (uint32_t q = use_off[s], e = use_off[s + 1]; q < e; q++) {
    const uint32_t d = cdef[q];
    if (d != ~0u) gslot[goff[d] + atomicSub(ccnt + d, 1u) - 1u] = (uint32_t)s;
  }
}

// ------------------------------------------------------------------------------------------ D
// Threads [0, nc) finish candidate c's trace if it left its window (k_resolve traced the in-window
// steps) and record store roots (R8); threads [nc, 2nc) update the key-group statistics of
// candidate c - nc (two independent latency chains per candidate run on different threads).
__global__ void k_trace(const Rec* __restrict__ rec, const KDesc* __restrict__ kd, const uint32_t* __restrict__ ptrrd,
                        uint64_t nc, uint32_t D, CandArrays ca, GroupTable gt, gs_kernel_stats* kst) {
  __shared__ uint16_t s_cls[OP_COUNT];
  pdl_trigger();
  opcls_init(s_cls);
  __syncthreads();
  const uint64_t t = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (t >= 2 * nc) return;
  const bool groups = t >= nc;
  const uint64_t c = groups ? t - nc : t;
  if (!groups) {
    uint32_t tk = ca.tk[c];
    if (tk == GS_T_NONE) return;
    const uint32_t kernel = ca.kernel[c];
    const uint32_t op = r_op(ld_rec(ca.rec, c)), cls = s_cls[op];
    uint32_t tv = ca.tv[c];
    if (tk == kTCont) {
      const KDesc K = kd[kernel];
      uint32_t n = ca.depth[c];
      const TraceOut tr = chase_from(rec, ptrrd, K, tv, ca.cont[c], n, D, 0, s_cls, [&](uint32_t j) {
        if (n < kChain4) ca.chain4[c * kChain4 + n] = j;
        n++;
      });
      tk = tr.tk;
      tv = tr.tv;
      ca.tk[c] = (uint8_t)tk;
      ca.tv[c] = tv;
      ca.depth[c] = (uint8_t)tr.depth;
    }
    if (cls & C_STORE) {  // store roots (R8, R27)
      if (tk == GS_T_PARAM || tk == GS_T_ENTRY) {
        const KHash H = gt.kh[kernel];
        hinsert<1>(gt.r + H.rofs, H.rmask, root_key(kernel, tk, tv));
      } else {
        atomicAdd(&kst[kernel].n_unresolved_stores, 1u);
      }
    }
    return;
  }
  const uint32_t kernel = ca.kernel[c];
  const Rec ri = ld_rec(ca.rec, c);
  const uint32_t op = r_op(ri), cls = s_cls[op];
  const bool traced = (cls & C_TRACED) && (r_flags(ri) & F_HASMEM);
  const uint32_t base = r_s0(ri), brd = ca.base_rd[c];
  const bool act = traced && op == OP_LDG;
  // key-group statistics (R3): n_loads, distinct offsets (all / 32-bit), min, max, contiguity.
  // Consecutive loads off one base definition (an unrolled loop body) share a group: the lanes of a
  // warp with the same key insert it once and add their count with one atomic (the CAS probes were
  // this kernel's longest stall).
  const unsigned long long key = act ? group_key(base, brd, kernel) : ~0ull;
  const uint32_t am = __activemask(), lane = threadIdx.x & 31u;
  const uint32_t peers = __match_any_sync(am, key);
  const uint32_t leader = __ffs(peers) - 1;
  const KHash H = gt.kh[kernel];
  GEnt* G = gt.g + H.gofs;
  uint32_t slot = 0;
  if (act && lane == leader) {
    slot = hinsert<4>(&G->key, H.gmask, key);
    atomicAdd(&G[slot].nload, (uint32_t)__popc(peers));
  }
  slot = __shfl_sync(am, slot, leader);
  if (!act) {
    ca.grp[c] = 0xffffffffu;
    return;
  }
  ca.grp[c] = (uint32_t)(H.gofs + slot);
  GEnt* e = G + slot;
  const int32_t off = r_imm(ri);
  const bool is32 = r_aw(ri) == AW_32;
  OEnt* O = gt.o + H.gofs;
  const uint32_t os_slot = hinsert<2>(&O->key, H.gmask, ((unsigned long long)slot << 32) | (uint32_t)off);
  const uint32_t prev = atomicOr(&O[os_slot].flags, is32 ? 3u : 2u);
  if (!(prev & 2u)) atomicAdd(&e->nall, 1u);
  if (is32 && !(prev & 1u)) {
    atomicAdd(&e->n32, 1u);
    atomicMin(&e->mn, off);
    atomicMax(&e->mx, off);
    atomicOr(&e->bits, (uint32_t)off & 3u);
    atomicAnd(&e->bits, ((((uint32_t)off & 3u) << 2) | 3u));
  }
}

// ------------------------------------------------------------------------------------------ E
struct RuleCfg {
  uint32_t TA, TL;
};

__device__ uint32_t eval_rules(const Rec& ri, uint64_t c, const CandArrays& ca, const GroupTable& gt,
                               const uint32_t* narith, RuleCfg rc, const uint16_t* cls_tab) {
  const uint32_t op = r_op(ri), cls = cls_tab[op], fl = r_flags(ri);
  uint32_t f = 0;
  if (!(fl & F_HASMEM) && !(cls & C_CONV)) return 0;
  if (op == OP_LDG && (fl & F_HASMEM)) {
    const GEnt& e = gt.g[ca.grp[c]];
    const uint32_t n32 = e.n32, nall = e.nall, nload = e.nload;
    if (r_aw(ri) == AW_32 && n32 >= 2) f |= 1u << GS_VEC;                                // O6
    if (narith[ca.idx[c]] >= rc.TA && (nload >= rc.TL || ca.ld[c] >= 1)) f |= 1u << GS_SHMEM;  // O8
    const uint32_t tk = ca.tk[c];
    bool ro = !(fl & F_CONSTANT) && (tk == GS_T_PARAM || tk == GS_T_ENTRY);
    if (ro) {
      const uint32_t k = ca.kernel[c];
      const KHash H = gt.kh[k];
      ro = !hcontains(gt.r + H.rofs, H.rmask, root_key(k, tk, ca.tv[c]));              // O10
    }
    if (ro) f |= 1u << GS_RO;
    if (ro && nall >= 2) f |= 1u << GS_TEX;                                              // O11
  }
  if ((op == OP_STL || op == OP_LDL) && (fl & F_HASMEM)) f |= 1u << GS_SPILL;          // O7
  if ((cls & C_GATOM) && (fl & F_HASMEM)) f |= 1u << GS_GATOM;                         // O9
  if (cls & C_CONV) f |= 1u << GS_CONV;                                                // O12
  return f;
}

// Site and chain-pool compaction (a-7) without separate scan passes: k_rules leaves one packed
// (chains << 32 | sites) sum per 256-candidate tile, one CTA scans the tile sums, and k_write
// re-derives each candidate's offsets inside its tile with a block scan.
constexpr int kCT = 256;  // candidates per tile (k_rules / k_write CTA)

__device__ __forceinline__ unsigned long long warp_incl64(unsigned long long v) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long x = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += x;
  }
  return v;
}
// exclusive scan over the CTA of one value per thread (blockDim.x = NT); *total = the CTA's sum
template <int NT>
__device__ __forceinline__ unsigned long long block_excl64(unsigned long long v, unsigned long long* total) {
  __shared__ unsigned long long wsum[NT / 32];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const unsigned long long inc = warp_incl64(v);
  if (lane == 31) wsum[warp] = inc;
  __syncthreads();
  if (warp == 0) {
    unsigned long long x = lane < NT / 32 ? wsum[lane] : 0;
    x = warp_incl64(x);
    if (lane < NT / 32) wsum[lane] = x;
  }
  __syncthreads();
  const unsigned long long before = warp ? wsum[warp - 1] : 0;
  *total = wsum[NT / 32 - 1];
  __syncthreads();
  return before + inc - v;
}
// per candidate: sites (low 32 bits) and chain-pool entries (high 32 bits); a tile's sums fit
__device__ __forceinline__ unsigned long long site_chain(uint32_t f, uint32_t depth) {
  return ((unsigned long long)(f ? depth : 0u) << 32) | (unsigned long long)__popc(f);
}

__global__ void __launch_bounds__(kCT) k_rules(const Rec* __restrict__ rec, uint64_t nc, CandArrays ca, GroupTable gt,
                                               const uint32_t* __restrict__ narith, RuleCfg rc,
                                               unsigned long long* __restrict__ tsum) {
  __shared__ uint16_t s_cls[OP_COUNT];
  opcls_init(s_cls);
  pdl_wait();
  pdl_trigger();
  __syncthreads();
  const uint64_t c = blockIdx.x * (uint64_t)kCT + threadIdx.x;
  unsigned long long v = 0;
  if (c < nc) {
    const Rec ri = ld_rec(ca.rec, c);
    const uint32_t f = eval_rules(ri, c, ca, gt, narith, rc, s_cls);
    ca.flags[c] = (uint8_t)f;
    v = site_chain(f, ca.depth[c]);
  }
  unsigned long long tot;
  block_excl64<kCT>(v, &tot);
  if (threadIdx.x == 0) tsum[blockIdx.x] = tot;
}

// one CTA: exclusive prefixes of the tile sums, sites and chains as separate u64 counters;
// tot[0] = chain-pool entries, tot[1] = sites. Warp w owns a contiguous segment of the tiles: its
// lanes sum the segment with coalesced loads, one warp scans the 32 segment totals, then each
// warp re-reads its segment 32 tiles at a time and writes the prefixes (warp scans, no barriers
// per tile group).
__device__ __forceinline__ void warp_incl_pair(unsigned long long& a, unsigned long long& b) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long x = __shfl_up_sync(0xffffffffu, a, o), y = __shfl_up_sync(0xffffffffu, b, o);
    if (lane >= o) { a += x; b += y; }
  }
}
__global__ void __launch_bounds__(1024) k_tile_prefix(const unsigned long long* __restrict__ tsum, uint64_t nt,
                                                      unsigned long long* __restrict__ pre_s,
                                                      unsigned long long* __restrict__ pre_c,
                                                      unsigned long long* __restrict__ tot) {
  __shared__ unsigned long long ws[32], wc[32];
  pdl_wait();
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  const uint64_t seg = (nt + 31) / 32, a = min(nt, warp * seg), e = min(nt, a + seg);
  unsigned long long ls = 0, lc = 0;
  for (uint64_t i = a + lane; i < e; i += 32) {
    const unsigned long long v = tsum[i];
    ls += v & 0xffffffffull;
    lc += v >> 32;
  }
  for (int o = 16; o; o >>= 1) {
    ls += __shfl_xor_sync(0xffffffffu, ls, o);
    lc += __shfl_xor_sync(0xffffffffu, lc, o);
  }
  if (lane == 0) { ws[warp] = ls; wc[warp] = lc; }
  __syncthreads();
  if (warp == 0) {
    unsigned long long x = ws[lane], y = wc[lane];
    const unsigned long long x0 = x, y0 = y;
    warp_incl_pair(x, y);
    ws[lane] = x - x0;  // exclusive prefix of segment `lane`
    wc[lane] = y - y0;
    if (lane == 31) { tot[0] = y; tot[1] = x; }
  }
  __syncthreads();
  unsigned long long rs = ws[warp], rc = wc[warp];  // running prefix of this warp's segment
  for (uint64_t i0 = a; i0 < e; i0 += 32) {
    const uint64_t i = i0 + lane;
    const unsigned long long v = i < e ? tsum[i] : 0ull;
    unsigned long long s_ = v & 0xffffffffull, c_ = v >> 32;
    warp_incl_pair(s_, c_);
    if (i < e) {
      pre_s[i] = rs + s_ - (v & 0xffffffffull);
      pre_c[i] = rc + c_ - (v >> 32);
    }
    rs += __shfl_sync(0xffffffffu, s_, 31);
    rc += __shfl_sync(0xffffffffu, c_, 31);
  }
}

__global__ void __launch_bounds__(kCT) k_write(const Rec* __restrict__ rec, const KDesc* __restrict__ kd,
                                               const uint32_t* __restrict__ ptrrd, uint64_t nc, uint32_t D, CandArrays ca,
                                               GroupTable gt, const uint32_t* __restrict__ narith,
                                               const unsigned long long* __restrict__ pre_s,
                                               const unsigned long long* __restrict__ pre_c, gs_site* __restrict__ sites,
                                               uint32_t* __restrict__ chain, uint64_t site_cap, uint64_t chain_cap) {
  // Launched before the host knows the totals: writes past the buffers' current capacities are
  // skipped, and the host relaunches after growing them when a total exceeds its capacity.
  __shared__ uint16_t s_cls[OP_COUNT];
  opcls_init(s_cls);  // (block_excl64 below synchronises the CTA before the first use)
  const uint64_t c = blockIdx.x * (uint64_t)kCT + threadIdx.x;
  const uint32_t f = c < nc ? ca.flags[c] : 0u;
  unsigned long long tot;
  const unsigned long long ex = block_excl64<kCT>(site_chain(f, c < nc ? ca.depth[c] : 0u), &tot);
  if (!f) return;
  const uint32_t g = ca.idx[c], kernel = ca.kernel[c];
  const KDesc K = kd[kernel];
  const Rec ri = ld_rec(ca.rec, c);
  const unsigned long long coff = pre_c[blockIdx.x] + (ex >> 32);
  // chain (kernel-local indices): the first kChain4 elements were kept by the trace; longer chains
  // are traced again
  const uint32_t dep = ca.depth[c];
  if (dep && coff + dep <= chain_cap) {
    if (dep <= kChain4) {
      const uint4 e = reinterpret_cast<const uint4*>(ca.chain4)[c];
      chain[coff] = e.x;
      if (dep > 1) chain[coff + 1] = e.y;
      if (dep > 2) chain[coff + 2] = e.z;
      if (dep > 3) chain[coff + 3] = e.w;
    } else {
      uint32_t n = 0;
      chase(rec, ptrrd, K, r_s0(ri), ca.base_rd[c], D, s_cls, [&](uint32_t j) { chain[coff + n++] = j; });
    }
  }
  uint64_t so = pre_s[blockIdx.x] + (ex & 0xffffffffull);
  for (uint32_t rule = 0; rule < 7; rule++) {
    if (!((f >> rule) & 1u)) continue;
    gs_site s;
    s.kernel = kernel;
    s.idx = g - K.first;
    s.rule = (uint8_t)rule;
    s.depth = ca.depth[c];
    s.term_kind = ca.tk[c];
    s.loop_depth = ca.ld[c];
    s.term_value = ca.tv[c];
    s.chain_off = (uint32_t)coff;
    s.a0 = s.a1 = s.a2 = 0;
    if (rule == GS_VEC) {
      const GEnt& e = gt.g[ca.grp[c]];
      const uint32_t n32 = e.n32;
      const int32_t mn = e.mn, mx = e.mx;
      const bool contig = (int64_t)mx - (int64_t)mn == 4ll * ((int64_t)n32 - 1) && (e.bits & 3u) == (e.bits >> 2);
      s.a0 = (int32_t)(n32 | (contig ? (1u << 30) : 0u));
      s.a1 = mn;
      s.a2 = mx;
    } else if (rule == GS_SPILL) {
      if (r_op(ri) == OP_STL) {
        s.a0 = (int32_t)r_s1(ri);
        const uint32_t rd = ca.data_rd[c];
        s.a1 = rd == 0xffffffffu ? -2 : (rd == 0 ? -1 : (int32_t)(rd - 1 - K.first));
      } else {
        s.a0 = (int32_t)r_dst(ri);
        s.a1 = -2;
      }
    } else if (rule == GS_SHMEM) {
      s.a0 = (int32_t)gt.g[ca.grp[c]].nload;
      s.a1 = (int32_t)narith[g];
    } else if (rule == GS_TEX) {
      s.a0 = (int32_t)gt.g[ca.grp[c]].nall;
    }
    if (rule == GS_CONV) { s.depth = 0; s.term_kind = GS_T_NONE; s.term_value = 0; }
    if (so < site_cap) {  // two 16-byte stores (gs_site is 32 bytes, 32-byte aligned)
      static_assert(sizeof(gs_site) == 32, "site layout");
      uint4 v[2];
      memcpy(v, &s, 32);
      uint4* d = reinterpret_cast<uint4*>(sites + so);
      d[0] = v[0];
      d[1] = v[1];
    }
    so++;
  }
}


// entries [g0, g1) of the group and offset tables, [r0, r1) of the root table (the regions of the
// detected kernels); runs on a side stream, concurrently with k_summary .. k_resolve
__global__ void k_init_groups(GroupTable gt, uint64_t g0, uint64_t g1, uint64_t r0, uint64_t r1) {
  const uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x;
  if (g0 + i < g1) {
    GEnt e;
    e.key = kEmpty;
    e.nload = e.n32 = e.nall = 0;
    e.mn = INT_MAX;
    e.mx = INT_MIN;
    e.bits = 3u << 2;
    gt.g[g0 + i] = e;
    OEnt o;
    o.key = kEmpty;
    o.flags = o.pad = 0;
    gt.o[g0 + i] = o;
  }
  if (r0 + i < r1) gt.r[r0 + i] = kEmpty;
}

}  // namespace

void detect_free(gs_ctx* c) {
  void* ps[] = {c->d_tab, c->d_ldiff, c->d_wsum, c->d_wloop, c->d_wev, c->d_ptrrd, c->d_narith,
                c->cand.idx, c->cand.kernel, c->cand.base_rd, c->cand.data_rd, c->cand.tv, c->cand.grp,
                c->cand.cont, c->cand.rec, c->cand.chain4, c->cand.ld, c->cand.tk, c->cand.depth, c->cand.flags,
                c->cand.choff, c->grp.g, c->grp.o, c->grp.r, c->grp.kh, c->d_kstats, c->d_sites,
                c->d_chain, c->d_scan_tmp};
  for (void* p : ps)
    if (p) cudaFree(p);
  c->d_tab = nullptr; c->d_ldiff = nullptr; c->d_wsum = nullptr; c->d_wloop = nullptr; c->d_wev = nullptr;
  c->d_ptrrd = nullptr; c->d_narith = nullptr;
  c->cand = CandArrays();
  c->grp = GroupTable();
  c->d_kstats = nullptr;
  c->d_sites = nullptr; c->sites_cap = 0; c->n_sites = 0;
  c->d_chain = nullptr; c->chain_cap = 0; c->n_chain = 0;
  c->d_scan_tmp = nullptr; c->scan_tmp_bytes = 0;
  void* cp[] = {c->d_cdef, c->d_ccnt, c->d_cgoff, c->d_cgslot, c->d_ctot};
  for (void* p : cp)
    if (p) cudaFree(p);
  c->d_cdef = c->d_ccnt = c->d_cgoff = c->d_cgslot = nullptr;
  c->d_ctot = nullptr;
  c->cdef_cap = c->ccnt_cap = c->cgoff_cap = c->cgslot_cap = 0;
  c->cons_ready = false;
  if (c->det_exec) cudaGraphExecDestroy(c->det_exec);
  c->det_exec = nullptr;
  c->det_key.clear();
  c->detected = false;
  c->det_pending = false;
}

// GS_JOIN_CONSUMER: consumer groups of the slots of kernels [kb, ke) (R37)
gs_status consumers_run(gs_ctx* c, uint32_t kb, uint32_t ke, uint32_t w0, uint32_t nw) {
  cudaStream_t st = c->stream;
  c->cons_ready = false;
  const uint64_t s0 = kb < c->n_kernels ? c->kd_h[kb].first : c->n_instr;
  const uint64_t s1 = ke < c->n_kernels ? c->kd_h[ke].first : c->n_instr;
  const uint64_t n = s1 - s0;
  gs_status us = uses_upload(c);
  if (us != GS_OK) return us;
  const uint64_t nuse = c->use_off_h.empty() ? 0 : c->use_off_h.back();
  GS_CUDA(c, dev_grow(&c->d_cdef, &c->cdef_cap, nuse ? nuse : 1));
  GS_CUDA(c, dev_grow(&c->d_ccnt, &c->ccnt_cap, c->n_instr + 1));
  GS_CUDA(c, dev_grow(&c->d_cgoff, &c->cgoff_cap, c->n_instr + 1));
  GS_CUDA(c, dev_grow(&c->d_cgslot, &c->cgslot_cap, n + (c->use_off_h[s1] - c->use_off_h[s0]) + 1));
  if (!c->d_ctot) GS_CUDA(c, cudaMalloc((void**)&c->d_ctot, 8));
  k_cons_init<<<(unsigned)((n + 1 + 255) / 256), 256, 0, st>>>(c->d_ccnt, s0, n); count_launch();
  if (nw) {
    k_consumers<<<(nw + kWarps - 1) / kWarps, kWarps * 32, 0, st>>>(c->d_rec, c->d_wd, w0, nw, c->d_tab, c->d_use_off,
                                                                    c->d_use_reg, c->d_cdef, c->d_ccnt); count_launch();
  }
  GS_CUDA(c, cudaGetLastError());
  us = scan_u32(c, c->d_ccnt + s0, c->d_cgoff + s0, n + 1, c->d_ctot);
  if (us != GS_OK) return us;
  if (n) {
    k_cons_fill<<<(unsigned)((n + 255) / 256), 256, 0, st>>>(s0, n, c->d_use_off, c->d_cdef, c->d_cgoff, c->d_ccnt,
                                                            c->d_cgslot); count_launch();
    GS_CUDA(c, cudaGetLastError());
  }
  c->cons_ready = true;
  return GS_OK;
}

gs_status detect_alloc(gs_ctx* c) {
  const uint64_t P = c->n_instr, NW = c->n_win, NC = c->n_cand ? c->n_cand : 1;
#define A(ptr, bytes) GS_CUDA(c, cudaMalloc((void**)&(ptr), (bytes) ? (bytes) : 16))
  A(c->d_tab, NW * kNumRegs * 4);
  A(c->d_ldiff, P * 4);
  GS_CUDA(c, cudaMemsetAsync(c->d_ldiff, 0, P * 4, c->stream));
  A(c->d_wsum, NW * 4);
  A(c->d_wloop, NW * 4);
  A(c->d_wev, NW * 4);
  A(c->d_ptrrd, P * 4);
  A(c->d_narith, P * 4);
  A(c->cand.idx, NC * 4); A(c->cand.kernel, NC * 4); A(c->cand.base_rd, NC * 4); A(c->cand.data_rd, NC * 4);
  A(c->cand.tv, NC * 4); A(c->cand.grp, NC * 4); A(c->cand.cont, NC * 4); A(c->cand.rec, NC * sizeof(Rec)); A(c->cand.chain4, NC * 16);
  A(c->cand.ld, NC); A(c->cand.tk, NC); A(c->cand.depth, NC); A(c->cand.flags, NC);
  A(c->cand.choff, 24 * ((NC + kCT - 1) / kCT) + 16);  // tile sums, prefixes, totals (k_rules / k_write)
  A(c->grp.g, c->grp.gtot * sizeof(GEnt));
  A(c->grp.o, c->grp.gtot * sizeof(OEnt));
  A(c->grp.r, c->grp.rtot * 8);
  A(c->grp.kh, (uint64_t)c->kh_h.size() * sizeof(KHash));
  if (!c->kh_h.empty())
    GS_CUDA(c, cudaMemcpyAsync(c->grp.kh, c->kh_h.data(), c->kh_h.size() * sizeof(KHash), cudaMemcpyHostToDevice,
                               c->stream));
  A(c->d_kstats, (uint64_t)(c->n_kernels ? c->n_kernels : 1) * sizeof(gs_kernel_stats));
#undef A
  return GS_OK;
}

// a launch whose grid may start while the previous kernel on the stream drains (the kernel waits
// for it with pdl_wait before reading its outputs)
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*k)(KArgs...), uint32_t grid, uint32_t block, cudaStream_t st, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.stream = st;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = 1;
#ifndef GS_NO_PDL
  cfg.attrs = at;
  cfg.numAttrs = 1;
#endif
  return cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

// k_write over the candidates of the last detection (also the relaunch after growing the buffers)
static gs_status write_launch(gs_ctx* c) {
  const uint64_t nc = c->det_nc, ntile = (nc + kCT - 1) / kCT;
  if (!nc || (!c->sites_cap && !c->chain_cap)) return GS_OK;
  unsigned long long* d_pre_s = c->cand.choff + ntile;
  unsigned long long* d_pre_c = d_pre_s + ntile;
  k_write<<<(uint32_t)ntile, kCT, 0, c->stream>>>(c->d_rec, c->d_kd, c->d_ptrrd, nc, c->det_D, c->cand, c->grp,
                                                   c->d_narith, d_pre_s, d_pre_c, c->d_sites, c->d_chain,
                                                   c->sites_cap, c->chain_cap);
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

// the host half of a detection: read the totals and counters, grow the buffers and write again if
// a total exceeded them
gs_status detect_finish(gs_ctx* c) {
  if (!c->det_pending) return GS_OK;
  c->det_pending = false;
  cudaStream_t st = c->stream;
  GS_CUDA(c, cudaStreamSynchronize(st));
  const unsigned long long* tot = static_cast<const unsigned long long*>(c->h_det);
  const gs_kernel_stats* kst_pin = reinterpret_cast<const gs_kernel_stats*>(static_cast<const char*>(c->h_det) + 16);
  c->kstats_h.assign(kst_pin, kst_pin + c->n_kernels);
  const uint64_t ns = tot[1], nch = tot[0];
  if (nch > 0xffffffffull) {
    c->detected = false;
    return fail(c, GS_E_RANGE, "chain pool exceeds 2^32 entries");
  }
  if (ns > c->sites_cap || nch > c->chain_cap) {
    GS_CUDA(c, dev_grow(&c->d_sites, &c->sites_cap, ns ? ns : 1));
    GS_CUDA(c, dev_grow(&c->d_chain, &c->chain_cap, nch ? nch : 1));
    const gs_status ws = write_launch(c);
    if (ws != GS_OK) return ws;
    GS_CUDA(c, cudaStreamSynchronize(st));
  }
  c->n_sites = ns;
  c->n_chain = nch;
  return GS_OK;
}

gs_status detect_run(gs_ctx* c, uint32_t kb, uint32_t ke, uint64_t* n_sites) {
  {  // a previous asynchronous detection's results are read before its buffers are reused
    const gs_status fs = detect_finish(c);
    if (fs != GS_OK) return fs;
  }
  cudaStream_t st = c->stream;
  const uint32_t w0 = kb < c->n_kernels ? c->kd_h[kb].win0 : c->n_win;
  const uint32_t w1 = ke < c->n_kernels ? c->kd_h[ke].win0 : c->n_win;
  const uint32_t nw = w1 - w0;
  const uint64_t c0 = c->cbase_h[w0], c1 = c->cbase_h[w1], nc = c1 - c0;
  const uint32_t D = c->cfg.trace_depth;
  c->detected = false;
  const bool cons = c->cfg.join_mode == GS_JOIN_CONSUMER;
  if (!c->side_stream) {
    GS_CUDA(c, cudaStreamCreateWithFlags(&c->side_stream, cudaStreamNonBlocking));
    GS_CUDA(c, cudaEventCreateWithFlags(&c->ev_fork, cudaEventDisableTiming));
    GS_CUDA(c, cudaEventCreateWithFlags(&c->ev_join, cudaEventDisableTiming));
  }
  // tile sums, their exclusive prefixes (sites, chains) and the two totals, carved from cand.choff
  // (3 x ceil(NC / 256) u64 + 2)
  const uint64_t ntile = (nc + kCT - 1) / kCT;
  unsigned long long* d_tsum = c->cand.choff;
  unsigned long long* d_pre_s = d_tsum + ntile;
  unsigned long long* d_pre_c = d_pre_s + ntile;
  unsigned long long* d_tot = d_pre_c + ntile;
  // pinned: [0, 16) the two totals, then the per-kernel counters (async D2H, one synchronisation)
  {
    const size_t need = 16 + (size_t)c->n_kernels * sizeof(gs_kernel_stats);
    if (!c->h_det || c->h_det_bytes < need) {
      if (c->h_det) cudaFreeHost(c->h_det);
      c->h_det = nullptr;
      c->h_det_bytes = 0;
      GS_CUDA(c, cudaHostAlloc(&c->h_det, need < 4096 ? 4096 : need, cudaHostAllocDefault));
      c->h_det_bytes = need < 4096 ? 4096 : need;
    }
  }
  unsigned long long* tot = static_cast<unsigned long long*>(c->h_det);
  gs_kernel_stats* kst_pin = reinterpret_cast<gs_kernel_stats*>(static_cast<char*>(c->h_det) + 16);
  tot[0] = tot[1] = 0;
  c->det_nc = nc;
  c->det_D = D;
  // sites and chains into the buffers as they are (one host synchronisation per call); if a total
  // turns out larger than its buffer, grow it and write again
  // sites and chains into the buffers as they are (one host synchronisation per call); if a total
  // turns out larger than its buffer, detect_finish grows it and writes again
  auto write = [&]() -> gs_status { return write_launch(c); };
  // everything up to the speculative write and the read-backs (no allocation in here)
  const auto enqueue = [&]() -> gs_status {
    if (nc) {  // the hash-table regions of kernels [kb, ke), zeroed on a side stream meanwhile
      const uint64_t g0 = c->kh_h[kb].gofs, r0 = c->kh_h[kb].rofs;
      const uint64_t g1 = ke < c->n_kernels ? c->kh_h[ke].gofs : c->grp.gtot;
      const uint64_t r1 = ke < c->n_kernels ? c->kh_h[ke].rofs : c->grp.rtot;
      const uint64_t ni = std::max(g1 - g0, r1 - r0);
      GS_CUDA(c, cudaEventRecord(c->ev_fork, st));
      GS_CUDA(c, cudaStreamWaitEvent(c->side_stream, c->ev_fork, 0));
      k_init_groups<<<(uint32_t)((ni + 255) / 256), 256, 0, c->side_stream>>>(c->grp, g0, g1, r0, r1);
      count_launch();
      GS_CUDA(c, cudaGetLastError());
      GS_CUDA(c, cudaEventRecord(c->ev_join, c->side_stream));
    }
    GS_CUDA(c, cudaMemsetAsync(c->d_kstats, 0, (uint64_t)c->n_kernels * sizeof(gs_kernel_stats), st));
    if (nw) {
      GS_CUDA(c, cudaMemsetAsync(c->d_wsum + w0, 0, (uint64_t)nw * 4, st));
      GS_CUDA(c, cudaMemsetAsync(c->d_wev + w0, 0, (uint64_t)nw * 4, st));
      const uint32_t grid = (nw + kWarps - 1) / kWarps;
      k_summary<<<grid, kWarps * 32, 0, st>>>(c->d_rec, c->d_wd, c->d_kd, w0, nw, c->d_tab, c->d_ldiff, c->d_wsum,
                                             c->d_wev, c->d_narith, c->d_kstats, c->win); count_launch();
      GS_CUDA(c, cudaGetLastError());
      GS_CUDA(c, launch_pdl(k_carry, ke - kb, 352, st, c->d_kd, kb, ke, c->d_tab, c->d_wsum, c->d_wloop, c->win));
      count_launch();
      // candidate arrays are indexed relative to c0
      GS_CUDA(c, launch_pdl(k_resolve, grid, kWarps * 32, st, c->d_rec, c->d_wd, c->d_kd, w0, nw, c->d_tab, c->d_ldiff,
                            c->d_wloop, c->d_wev, c->d_cbase, c0, c->d_ptrrd, c->d_narith, c->cand, D));
      count_launch();
      GS_CUDA(c, cudaGetLastError());
    }
    if (cons) {
      const gs_status cs = consumers_run(c, kb, ke, w0, nw);
      if (cs != GS_OK) return cs;
    }
    if (nc) {
      GS_CUDA(c, cudaStreamWaitEvent(st, c->ev_join, 0));
      const uint32_t gridc = (uint32_t)((nc + 255) / 256);
      k_trace<<<2 * gridc, 256, 0, st>>>(c->d_rec, c->d_kd, c->d_ptrrd, nc, D, c->cand, c->grp, c->d_kstats);
      count_launch();
      GS_CUDA(c, cudaGetLastError());
      GS_CUDA(c, launch_pdl(k_rules, (uint32_t)ntile, kCT, st, c->d_rec, nc, c->cand, c->grp, c->d_narith,
                            RuleCfg{c->cfg.shmem_min_arith, c->cfg.shmem_min_loads}, d_tsum));
      count_launch();
      GS_CUDA(c, launch_pdl(k_tile_prefix, 1u, 1024u, st, d_tsum, ntile, d_pre_s, d_pre_c, d_tot)); count_launch();
      GS_CUDA(c, cudaGetLastError());
      GS_CUDA(c, cudaMemcpyAsync(tot, d_tot, 16, cudaMemcpyDeviceToHost, st));
    }
    gs_status ws = write();
    if (ws != GS_OK) return ws;
    if (c->n_kernels)
      GS_CUDA(c, cudaMemcpyAsync(kst_pin, c->d_kstats, (uint64_t)c->n_kernels * sizeof(gs_kernel_stats),
                                 cudaMemcpyDeviceToHost, st));
    return GS_OK;
  };
  c->cons_ready = false;
  // Replayed as one CUDA graph while (kernel range, buffers, capacities) repeat; not with the
  // consumer join (it allocates), nor on the default streams (not capturable).
  const uintptr_t key[] = {kb, ke, (uintptr_t)nc, D, (uintptr_t)c->sites_cap, (uintptr_t)c->chain_cap,
                           (uintptr_t)c->d_sites, (uintptr_t)c->d_chain, (uintptr_t)c->h_det,
                           c->cfg.shmem_min_arith, c->cfg.shmem_min_loads, (uintptr_t)c->n_kernels};
  constexpr size_t nkey = sizeof(key) / sizeof(key[0]);
  static const bool no_graph = getenv("GS_NO_GRAPH") != nullptr;
  const bool capturable = st != nullptr && st != cudaStreamLegacy && st != cudaStreamPerThread;
  if (!no_graph && !cons && capturable) {
    bool hit = c->det_exec && c->det_key.size() == nkey;
    for (size_t q = 0; hit && q < nkey; q++) hit = c->det_key[q] == key[q];
    if (!hit) {
      if (c->det_exec) cudaGraphExecDestroy(c->det_exec);
      c->det_exec = nullptr;
      const uint64_t l0 = launch_count_now();
      GS_CUDA(c, cudaStreamBeginCapture(st, cudaStreamCaptureModeThreadLocal));
      const gs_status s1 = enqueue();
      cudaGraph_t g = nullptr;
      const cudaError_t e = cudaStreamEndCapture(st, &g);
      if (s1 != GS_OK) {
        if (g) cudaGraphDestroy(g);
        return s1;
      }
      GS_CUDA(c, e);
      const cudaError_t ei = cudaGraphInstantiate(&c->det_exec, g, 0);
      cudaGraphDestroy(g);
      GS_CUDA(c, ei);
      c->det_key.assign(key, key + nkey);
      c->det_graph_launches = launch_count_now() - l0;
      count_launch_undo(c->det_graph_launches);
    }
    GS_CUDA(c, cudaGraphLaunch(c->det_exec, st));
    count_launch(c->det_graph_launches);
  } else {
    const gs_status s1 = enqueue();
    if (s1 != GS_OK) return s1;
  }
  c->det_kb = kb; c->det_ke = ke; c->det_c0 = c0; c->det_c1 = c1;
  c->detected = true;
  c->det_pending = true;
  if (!n_sites) return GS_OK;  // asynchronous: the next call that needs the results finishes it
  const gs_status fs = detect_finish(c);
  if (fs != GS_OK) return fs;
  *n_sites = c->n_sites;
  return GS_OK;
}

}  // namespace gs
