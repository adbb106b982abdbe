// liveness.cu — register pressure per SASS instruction ("the number
// of additional registers needed by each SASS instruction").
//
// Live general-purpose registers (R0..R254, 256-bit sets of 8 words) by backward dataflow over
// each kernel's control-flow graph (R36, with the sm_100a register forms and call ABI of
// R38: defs = the destination(s) of the record, plus the clobbered registers of a CALL below the
// kernel's register count; a RET reads the callee-saved registers; an indirect branch (BRX)
// continues at each target of its list):
//   live_in(i) = uses(i) | (live_out(i) & keep(i)),  keep(i) = guarded(i) ? all : ~defs(i)
//   count(i)   = |live_in(i) | defs(i)|  (+ R1, the stack pointer, after its first definition)
// The transfer function of an instruction, x -> U | (x & K), composes associatively:
//   (U1, K1) o (U2, K2) = (U1 | (U2 & K1), K1 & K2),
// so each basic block is summarised by one (U, K) pair (one thread per block), the fixed point is
// iterated over blocks only (one warp per kernel, lanes = bitset words), and a last pass walks
// every block backward from its live-out to write the per-instruction counts.
//
//   k_lv_leader   per kernel CTA: block leaders (first instruction, branch targets, after a branch
//                 or EXIT/RET)
//   scan          leader flags -> block ids
//   k_lv_blocks   block start slot and kernel; per-kernel first block
//   k_lv_transfer per block: (U, K), successors, IN = U; per kernel: first definition of R1
//   k_lv_fix      per kernel: round-robin (reverse block order) to the fixed point
//   k_lv_count    per block: counts of its instructions
#include <cuda_runtime.h>

#include <algorithm>

#include "ctx.h"

namespace gs {
namespace {

constexpr int kW = 8;  // 32-bit words per register set

struct LvScratch {
  uint32_t *leader, *excl, *bbstart, *bbkern, *kbb0, *r1def;
  uint32_t *U, *K, *IN;  // [nbb][kW]
  int32_t* succ;         // [nbb][2]: block ids; succ[2b] <= -2 means indirect-branch list -2 - succ[2b]
};

// indirect-branch successor lists (R38i): x -> kernel-local target indices [xoff[x], xoff[x+1])
struct XTargets {
  const uint32_t* off;
  const int32_t* tgt;
};

__device__ __forceinline__ void set_bit(uint32_t (&b)[kW], uint32_t r) {
#pragma unroll
  for (int w = 0; w < kW; w++)
    if ((r >> 5) == (uint32_t)w) b[w] |= 1u << (r & 31);
}

// registers [0, nregs) with call_clobbered(r) == clob (R38g), R1 excluded from the callee-saved set
__device__ __forceinline__ void abi_set(uint32_t (&b)[kW], uint32_t nregs, bool clob) {
  for (uint32_t r = 0; r < nregs && r < 255; r++)
    if (call_clobbered(r) == clob && (clob || r != 1)) set_bit(b, r);
}

// uses / defs / keep of the instruction at slot s
__device__ __forceinline__ void inst_sets(const Rec& rec, const uint32_t* __restrict__ use_off,
                                          const uint8_t* __restrict__ use_reg, uint64_t s, uint32_t nregs,
                                          uint32_t (&u)[kW], uint32_t (&d)[kW], uint32_t (&k)[kW]) {
#pragma unroll
  for (int w = 0; w < kW; w++) u[w] = d[w] = 0;
  for (uint32_t q = use_off[s], e = use_off[s + 1]; q < e; q++) set_bit(u, use_reg[q]);
  const uint32_t dst = r_dst(rec), dw = r_dstw(rec), dst2 = r_dst2(rec);
  if (dst < 255)
    for (uint32_t q = 0; q < dw && dst + q < 255; q++) set_bit(d, dst + q);
  if (dst2 < 255)
    for (uint32_t q = 0; q < dw && dst2 + q < 255; q++) set_bit(d, dst2 + q);
  const uint32_t op = r_op(rec);
  if (op == OP_CALL) abi_set(d, nregs, true);   // a call may overwrite the caller-saved registers
  if (op == OP_RET) abi_set(u, nregs, false);   // the caller reads the callee-saved ones back
  const bool guarded = r_flags(rec) & F_PRED;
#pragma unroll
  for (int w = 0; w < kW; w++) k[w] = guarded ? 0xffffffffu : ~d[w];
}

__device__ __forceinline__ bool valid_branch(const Rec& r, int32_t t, uint32_t n) {
  return r_op(r) == OP_BRA && t >= 0 && (uint32_t)t < n;
}
// an indirect branch with a target list (R38i)
__device__ __forceinline__ bool multi_branch(const Rec& r, int32_t t) { return r_op(r) == OP_BRX && t <= -2; }

__global__ void k_lv_leader(const Rec* __restrict__ rec, const int32_t* __restrict__ tgt,
                            const KDesc* __restrict__ kd, uint32_t kb, uint32_t s0, XTargets X,
                            uint32_t* __restrict__ leader) {
  const KDesc K = kd[kb + blockIdx.x];
  for (uint32_t i = threadIdx.x; i < K.n; i += blockDim.x) {
    const uint64_t s = (uint64_t)K.first + i;
    const Rec r = rec[s];
    const int32_t t = tgt[s];
    if (i == 0) leader[s - s0] = 1;
    const bool br = valid_branch(r, t, K.n), mb = multi_branch(r, t);
    if ((br || mb || (r_flags(r) & F_EXIT)) && i + 1 < K.n) leader[s + 1 - s0] = 1;
    if (br) leader[K.first + (uint32_t)t - s0] = 1;
    if (mb) {
      const uint32_t x = (uint32_t)(-2 - t);
      for (uint32_t q = X.off[x]; q < X.off[x + 1]; q++) leader[K.first + (uint32_t)X.tgt[q] - s0] = 1;
    }
  }
}

// word w of the live-in union of block b's successors
__device__ __forceinline__ uint32_t out_word(const LvScratch& L, const XTargets& X, uint32_t b, uint32_t first,
                                             uint32_t s0, int w) {
  const int32_t a = L.succ[2 * b], c = L.succ[2 * b + 1];
  uint32_t out = 0;
  if (a >= 0) out |= L.IN[(uint64_t)a * kW + w];
  else if (a <= -2)
    for (uint32_t q = X.off[-2 - a]; q < X.off[-1 - a]; q++)
      out |= L.IN[(uint64_t)L.excl[first + (uint32_t)X.tgt[q] - s0] * kW + w];
  if (c >= 0) out |= L.IN[(uint64_t)c * kW + w];
  return out;
}

__global__ void k_lv_blocks(const KDesc* __restrict__ kd, uint32_t kb, uint32_t s0, LvScratch L) {
  const uint32_t k = kb + blockIdx.x;
  const KDesc K = kd[k];
  for (uint32_t i = threadIdx.x; i < K.n; i += blockDim.x) {
    const uint32_t s = K.first + i - s0;
    if (L.leader[s]) {
      L.bbstart[L.excl[s]] = K.first + i;
      L.bbkern[L.excl[s]] = k;
    }
  }
  if (threadIdx.x == 0) {
    L.kbb0[blockIdx.x] = K.n ? L.excl[K.first - s0] : 0xffffffffu;
    L.r1def[blockIdx.x] = 0xffffffffu;
  }
}

__global__ void k_lv_transfer(const Rec* __restrict__ rec, const int32_t* __restrict__ tgt,
                              const uint32_t* __restrict__ use_off, const uint8_t* __restrict__ use_reg,
                              const KDesc* __restrict__ kd, uint32_t kb, uint32_t s0, uint32_t s1, uint32_t nbb,
                              LvScratch L) {
  const uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= nbb) return;
  const uint32_t start = L.bbstart[b], end = b + 1 < nbb ? L.bbstart[b + 1] : s1;
  const uint32_t k = L.bbkern[b];
  const KDesc Kd = kd[k];
  uint32_t U[kW], Kk[kW];
#pragma unroll
  for (int w = 0; w < kW; w++) { U[w] = 0; Kk[w] = 0xffffffffu; }
  uint32_t r1 = 0xffffffffu;
  for (uint32_t s = end; s-- > start;) {
    const Rec r = rec[s];
    uint32_t u[kW], d[kW], kp[kW];
    inst_sets(r, use_off, use_reg, s, kd_nregs(Kd), u, d, kp);
#pragma unroll
    for (int w = 0; w < kW; w++) {
      U[w] = u[w] | (U[w] & kp[w]);
      Kk[w] &= kp[w];
    }
    if (d[0] & 2u) r1 = s - Kd.first;
  }
  if (r1 != 0xffffffffu) atomicMin(&L.r1def[k - kb], r1);
  // successors of the block's last instruction
  const uint32_t e = end - 1, ie = e - Kd.first;
  const Rec r = rec[e];
  const int32_t t = tgt[e];
  const bool br = valid_branch(r, t, Kd.n), mb = multi_branch(r, t);
  const bool cond = r_flags(r) & (F_PRED | F_BRPRED);
  const bool stops = ((r_flags(r) & F_EXIT) || br || r_op(r) == OP_BRX) && !cond;
  L.succ[2 * b] = br ? (int32_t)L.excl[Kd.first + (uint32_t)t - s0] : (mb ? t : -1);
  L.succ[2 * b + 1] = (!stops && ie + 1 < Kd.n) ? (int32_t)(b + 1) : -1;
#pragma unroll
  for (int w = 0; w < kW; w++) {
    L.U[(uint64_t)b * kW + w] = U[w];
    L.K[(uint64_t)b * kW + w] = Kk[w];
    L.IN[(uint64_t)b * kW + w] = U[w];
  }
}

// one warp per kernel; lane w < kW owns word w of every set
__global__ void k_lv_fix(const KDesc* __restrict__ kd, uint32_t kb, uint32_t s0base, uint32_t nk, uint32_t nbb,
                         XTargets X, LvScratch L) {
  const uint32_t kk = blockIdx.x * (blockDim.x >> 5) + (threadIdx.x >> 5);
  if (kk >= nk) return;
  const uint32_t lane = threadIdx.x & 31u, w = lane & (kW - 1);
  const uint32_t b0 = L.kbb0[kk];
  if (b0 == 0xffffffffu) return;
  uint32_t b1 = nbb;
  for (uint32_t q = kk + 1; q < nk; q++)
    if (L.kbb0[q] != 0xffffffffu) { b1 = L.kbb0[q]; break; }
  const uint32_t first = kd[kb + kk].first;
  for (bool changed = true; changed;) {
    bool ch = false;
    for (uint32_t b = b1; b-- > b0;) {
      const uint32_t out = out_word(L, X, b, first, s0base, w);
      const uint32_t in = L.U[(uint64_t)b * kW + w] | (out & L.K[(uint64_t)b * kW + w]);
      if (lane < kW && in != L.IN[(uint64_t)b * kW + w]) {
        L.IN[(uint64_t)b * kW + w] = in;
        ch = true;
      }
      __syncwarp();
    }
    changed = __any_sync(0xffffffffu, ch);
  }
}

__global__ void k_lv_count(const Rec* __restrict__ rec, const uint32_t* __restrict__ use_off,
                           const uint8_t* __restrict__ use_reg, const KDesc* __restrict__ kd, uint32_t kb,
                           uint32_t s0base, uint32_t s1, uint32_t nbb, XTargets X, LvScratch L,
                           uint16_t* __restrict__ live) {
  const uint32_t b = blockIdx.x * blockDim.x + threadIdx.x;
  if (b >= nbb) return;
  const uint32_t start = L.bbstart[b], end = b + 1 < nbb ? L.bbstart[b + 1] : s1;
  const uint32_t k = L.bbkern[b];
  const KDesc Kd = kd[k];
  const uint32_t first = Kd.first, r1 = L.r1def[k - kb];
  uint32_t x[kW];
#pragma unroll
  for (int w = 0; w < kW; w++) x[w] = out_word(L, X, b, first, s0base, w);
  for (uint32_t s = end; s-- > start;) {
    uint32_t u[kW], d[kW], kp[kW];
    inst_sets(rec[s], use_off, use_reg, s, kd_nregs(Kd), u, d, kp);
    uint32_t c = 0;
#pragma unroll
    for (int w = 0; w < kW; w++) {
      x[w] = u[w] | (x[w] & kp[w]);
      c += __popc(x[w] | d[w]);
    }
    if (r1 != 0xffffffffu && s - first > r1 && !((x[0] | d[0]) & 2u)) c++;
    live[s] = (uint16_t)c;
  }
}

template <typename T>
T* carve(char*& p, uint64_t n) {
  T* r = reinterpret_cast<T*>(p);
  p += ((n * sizeof(T) + 255) / 256) * 256;
  return r;
}

}  // namespace

gs_status uses_upload(gs_ctx* c) {
  if (c->d_use_off) return GS_OK;  // first use: upload the packer's GPR use lists
  cudaStream_t st = c->stream;
  GS_CUDA(c, cudaMalloc((void**)&c->d_use_off, c->use_off_h.size() * 4));
  GS_CUDA(c, cudaMalloc((void**)&c->d_use_reg, std::max<size_t>(c->use_reg_h.size(), 1)));
  GS_CUDA(c, cudaMalloc((void**)&c->d_tgt, std::max<size_t>(c->tgt_h.size(), 1) * 4));
  GS_CUDA(c, cudaMalloc((void**)&c->d_xoff, c->xoff_h.size() * 4));
  GS_CUDA(c, cudaMalloc((void**)&c->d_xtgt, std::max<size_t>(c->xtgt_h.size(), 1) * 4));
  GS_CUDA(c, cudaMemcpyAsync(c->d_xoff, c->xoff_h.data(), c->xoff_h.size() * 4, cudaMemcpyHostToDevice, st));
  if (!c->xtgt_h.empty())
    GS_CUDA(c, cudaMemcpyAsync(c->d_xtgt, c->xtgt_h.data(), c->xtgt_h.size() * 4, cudaMemcpyHostToDevice, st));
  GS_CUDA(c, cudaMemcpyAsync(c->d_use_off, c->use_off_h.data(), c->use_off_h.size() * 4, cudaMemcpyHostToDevice, st));
  if (!c->use_reg_h.empty())
    GS_CUDA(c, cudaMemcpyAsync(c->d_use_reg, c->use_reg_h.data(), c->use_reg_h.size(), cudaMemcpyHostToDevice, st));
  if (!c->tgt_h.empty())
    GS_CUDA(c, cudaMemcpyAsync(c->d_tgt, c->tgt_h.data(), c->tgt_h.size() * 4, cudaMemcpyHostToDevice, st));
  return GS_OK;
}

gs_status liveness_run(gs_ctx* c, uint32_t kb, uint32_t ke, uint16_t* d_live) {
  cudaStream_t st = c->stream;
  if (ke <= kb) return GS_OK;
  const uint32_t s0 = c->kd_h[kb].first;
  const uint32_t s1 = ke < c->n_kernels ? c->kd_h[ke].first : (uint32_t)c->n_instr;
  const uint64_t n = s1 - s0, nk = ke - kb;
  if (!n) return GS_OK;
  {
    const gs_status us = uses_upload(c);
    if (us != GS_OK) return us;
  }
  // scratch sized for the worst case (every instruction a block): leader, excl, block arrays
  const uint64_t need = 8 * ((n * 4 + 255) / 256 * 256) + 3 * ((n * kW * 4 + 255) / 256 * 256) +
                        ((n * 8 + 255) / 256 * 256) + 2 * ((nk * 4 + 255) / 256 * 256) + 4096;
  if (c->lv_bytes < need) {
    if (c->d_lv) cudaFree(c->d_lv);
    c->d_lv = nullptr;
    c->lv_bytes = 0;
    GS_CUDA(c, cudaMalloc(&c->d_lv, need));
    c->lv_bytes = need;
  }
  char* p = static_cast<char*>(c->d_lv);
  LvScratch L;
  L.leader = carve<uint32_t>(p, n);
  L.excl = carve<uint32_t>(p, n);
  L.bbstart = carve<uint32_t>(p, n);
  L.bbkern = carve<uint32_t>(p, n);
  L.kbb0 = carve<uint32_t>(p, nk);
  L.r1def = carve<uint32_t>(p, nk);
  L.U = carve<uint32_t>(p, n * kW);
  L.K = carve<uint32_t>(p, n * kW);
  L.IN = carve<uint32_t>(p, n * kW);
  L.succ = carve<int32_t>(p, 2 * n);
  unsigned long long* d_total = carve<unsigned long long>(p, 1);
  const XTargets X{c->d_xoff, c->d_xtgt};
  GS_CUDA(c, cudaMemsetAsync(L.leader, 0, n * 4, st));
  k_lv_leader<<<(uint32_t)nk, 256, 0, st>>>(c->d_rec, c->d_tgt, c->d_kd, kb, s0, X, L.leader);
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  gs_status ss = scan_u32(c, L.leader, L.excl, n, d_total);
  if (ss != GS_OK) return ss;
  GS_CUDA(c, pin_grow(c, 8));
  unsigned long long* nbb_h = static_cast<unsigned long long*>(c->h_pin);
  GS_CUDA(c, cudaMemcpyAsync(nbb_h, d_total, 8, cudaMemcpyDeviceToHost, st));
  k_lv_blocks<<<(uint32_t)nk, 256, 0, st>>>(c->d_kd, kb, s0, L);
  count_launch();
  GS_CUDA(c, cudaStreamSynchronize(st));
  const uint32_t nbb = (uint32_t)*nbb_h;
  if (!nbb) return GS_OK;
  const uint32_t gb = (nbb + 127) / 128;
  k_lv_transfer<<<gb, 128, 0, st>>>(c->d_rec, c->d_tgt, c->d_use_off, c->d_use_reg, c->d_kd, kb, s0, s1, nbb, L);
  count_launch();
  k_lv_fix<<<(uint32_t)((nk + 3) / 4), 128, 0, st>>>(c->d_kd, kb, s0, (uint32_t)nk, nbb, X, L);
  count_launch();
  k_lv_count<<<gb, 128, 0, st>>>(c->d_rec, c->d_use_off, c->d_use_reg, c->d_kd, kb, s0, s1, nbb, X, L, d_live);
  count_launch();
  GS_CUDA(c, cudaGetLastError());
  return GS_OK;
}

void liveness_free(gs_ctx* c) {
  if (c->d_use_off) cudaFree(c->d_use_off);
  if (c->d_use_reg) cudaFree(c->d_use_reg);
  if (c->d_tgt) cudaFree(c->d_tgt);
  if (c->d_xoff) cudaFree(c->d_xoff);
  if (c->d_xtgt) cudaFree(c->d_xtgt);
  if (c->d_lv) cudaFree(c->d_lv);
  c->d_use_off = nullptr;
  c->d_use_reg = nullptr;
  c->d_tgt = nullptr;
  c->d_xoff = nullptr;
  c->d_xtgt = nullptr;
  c->d_lv = nullptr;
  c->lv_bytes = 0;
}

}  // namespace gs
