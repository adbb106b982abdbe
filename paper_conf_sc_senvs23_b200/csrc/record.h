// record.h — the packed 16-byte SASS instruction record and the opcode-class table of the GPU
// path (host packer + device kernels). Product code; shares nothing with oracle/.
//
// One record per instruction ("the instruction and the destination (+source) register numbers",
// P:211-213), laid out so a warp loads 32 consecutive records with one coalesced uint4 per lane.
//
//   w0: op[0:8) | flags[8:16) | aw[16:19) | pk[19:21) | cbank[21:26) | dstw[26:32) (low 6 bits)
//   w1: dst[0:9) | ptr[9:18) | s0[18:27) | dstw[27:29) (high 2 bits: widths up to 255, LDTM.x128)
//   w2: s1[0:9)  | s2[9:18)  | s3[18:27)
//   w3: imm (int32): memory offset / branch target (kernel-local index) / constant-bank offset
//
// Register ids (9 bits): GPR Rn -> n (RZ = 255), URn -> 256 + n (URZ = 319), none = 511.
// Memory instructions: s0 = address base register, s1 = stored/data register; a 256-bit load
// (LDG.E.ENL2.256 Ra, Rb, [..], R38a) carries its second destination quad Rb in s2 (F_DST2).
// ARITH instructions (R12): s0..s3 = register sources (RZ/URZ dropped, at most 4).
// pk = pointer-operand kind of the def-use trace step (R7): REG -> ptr register,
// CONST -> c[cbank][imm], IMM -> the trace ends at an immediate.
#pragma once
#include <stdint.h>

#ifdef __CUDACC__
#define GS_HD __host__ __device__ __forceinline__
#define GS_HDC __host__ __device__ constexpr
#else
#define GS_HD inline
#define GS_HDC constexpr
#endif

namespace gs {

constexpr int kRegNone = 511, kRZ = 255, kURZ = 319, kNumRegs = 320;
GS_HD bool reg_live(uint32_t r) { return r < 320u && r != 255u && r != 319u; }

enum Op : uint8_t {
  OP_OTHER = 0,
  OP_LDG, OP_LDL, OP_STL, OP_STG, OP_ST, OP_LD, OP_LDS, OP_STS, OP_LDSM,
  OP_ATOM, OP_ATOMG, OP_ATOMS, OP_RED, OP_REDG, OP_SUST, OP_SULD, OP_SUATOM,
  OP_TLD, OP_TLD4, OP_TLDS, OP_TEX, OP_TMML, OP_TXD, OP_TXQ, OP_LDTM,
  OP_LDC, OP_LDCU, OP_ULDC,
  OP_S2R, OP_S2UR, OP_CS2R,
  OP_BRA,
  OP_F2F, OP_F2I, OP_I2F, OP_I2I, OP_I2FP, OP_F2IP, OP_F2FP,
  OP_FADD, OP_FMUL, OP_FFMA, OP_FMNMX, OP_DADD, OP_DMUL, OP_DFMA, OP_HADD2, OP_HMUL2, OP_HFMA2,
  OP_MUFU, OP_IADD3, OP_VIADD, OP_IMAD, OP_IMUL, OP_IMNMX, OP_VIMNMX, OP_IABS,
  OP_IMAD_MOV, OP_LEA, OP_ULEA, OP_UIADD3, OP_UIMAD, OP_HMMA, OP_DMNMX, OP_FCHK,
  OP_CALL, OP_RET, OP_BRX,  // R38g/i: the call ABI and indirect branches (register pressure)
  OP_COUNT
};

// opcode classes
enum : uint32_t {
  C_ARITH = 1u << 0,      // R12
  C_CONV = 1u << 1,       // R16
  C_GATOM = 1u << 2,      // ATOMG ATOM RED REDG (O9)
  C_SATOM = 1u << 3,      // ATOMS
  C_STORE = 1u << 4,      // store-class roots for RO (R27)
  C_MEMLOAD = 1u << 5,    // trace terminal MEMORY (R26)
  C_CONSTLOAD = 1u << 6,  // trace terminal CONST/PARAM
  C_SREG = 1u << 7,       // trace terminal SREG
  C_BRA = 1u << 8,
  C_TRACED = 1u << 9,     // memory instruction whose address is traced (R27)
};

GS_HDC uint32_t op_class(uint32_t op) {
  switch (op) {
    case OP_LDG: return C_MEMLOAD | C_TRACED;
    case OP_LDL: return C_MEMLOAD | C_TRACED;
    case OP_STL: return C_TRACED;
    case OP_STG: case OP_ST: case OP_SUST: return C_STORE | C_TRACED;
    case OP_ATOM: case OP_ATOMG: return C_GATOM | C_STORE | C_MEMLOAD | C_TRACED;
    case OP_RED: case OP_REDG: return C_GATOM | C_STORE | C_TRACED;
    case OP_ATOMS: return C_SATOM | C_MEMLOAD;
    case OP_LD: case OP_LDS: case OP_LDSM: case OP_SULD: case OP_SUATOM: case OP_TLD: case OP_TLD4:
    case OP_TLDS: case OP_TEX: case OP_TMML: case OP_TXD: case OP_TXQ: case OP_LDTM:
      return C_MEMLOAD;
    case OP_LDC: case OP_LDCU: case OP_ULDC: return C_CONSTLOAD;
    case OP_S2R: case OP_S2UR: case OP_CS2R: return C_SREG;
    case OP_BRA: return C_BRA;
    case OP_F2F: case OP_F2I: case OP_I2F: case OP_I2I: case OP_I2FP: case OP_F2IP: case OP_F2FP:
      return C_CONV;
    case OP_FADD: case OP_FMUL: case OP_FFMA: case OP_FMNMX: case OP_DADD: case OP_DMUL: case OP_DFMA:
    case OP_HADD2: case OP_HMUL2: case OP_HFMA2: case OP_MUFU: case OP_IADD3: case OP_VIADD:
    case OP_IMAD: case OP_IMUL: case OP_IMNMX: case OP_VIMNMX: case OP_IABS:
      return C_ARITH;
    default: return 0;
  }
}

// flags
enum : uint32_t {
  F_CONSTANT = 1, F_HASMEM = 2, F_BRA_OK = 4,
  F_PRED = 8,     // guarded by a predicate other than PT (kills no register, R36)
  F_EXIT = 16,    // EXIT / RET
  F_BRPRED = 32,  // BRA with a predicate or register condition (BRA.U !UP0, BRA.DIV UR4; R38i)
  F_DST2 = 64,    // second destination quad in s2 (256-bit load, R38a)
};
// access width codes
enum : uint32_t { AW_NONE = 0, AW_8 = 1, AW_16 = 2, AW_32 = 3, AW_64 = 4, AW_128 = 5, AW_256 = 6 };
// pointer-operand kinds
enum : uint32_t { PK_IMM = 0, PK_REG = 1, PK_CONST = 2 };
// call ABI (R38g): registers a CALL may overwrite; the others (except R1) are callee-saved and live
// out of a RET
GS_HD bool call_clobbered(uint32_t r) { return r == 0 || (r >= 3 && r <= 15) || (r >= 32 && r <= 99 && (r - 32) % 8 < 4); }

struct Rec {
  uint32_t w0, w1, w2;
  int32_t w3;
};
static_assert(sizeof(Rec) == 16, "record is 16 bytes");

GS_HD uint32_t r_op(const Rec& r) { return r.w0 & 0xffu; }
GS_HD uint32_t r_flags(const Rec& r) { return (r.w0 >> 8) & 0xffu; }
GS_HD uint32_t r_aw(const Rec& r) { return (r.w0 >> 16) & 7u; }
GS_HD uint32_t r_pk(const Rec& r) { return (r.w0 >> 19) & 3u; }
GS_HD uint32_t r_cbank(const Rec& r) { return (r.w0 >> 21) & 31u; }
GS_HD uint32_t r_dstw(const Rec& r) { return (r.w0 >> 26) | (((r.w1 >> 27) & 3u) << 6); }
GS_HD uint32_t r_dst(const Rec& r) { return r.w1 & 511u; }
GS_HD uint32_t r_ptr(const Rec& r) { return (r.w1 >> 9) & 511u; }
GS_HD uint32_t r_s0(const Rec& r) { return (r.w1 >> 18) & 511u; }
GS_HD uint32_t r_s1(const Rec& r) { return r.w2 & 511u; }
GS_HD uint32_t r_s2(const Rec& r) { return (r.w2 >> 9) & 511u; }
GS_HD uint32_t r_s3(const Rec& r) { return (r.w2 >> 18) & 511u; }
GS_HD int32_t r_imm(const Rec& r) { return r.w3; }
// second destination quad of a 256-bit load (R38a), kRegNone otherwise
GS_HD uint32_t r_dst2(const Rec& r) { return (r_flags(r) & F_DST2) ? r_s2(r) : (uint32_t)kRegNone; }

GS_HD Rec make_rec(uint32_t op, uint32_t flags, uint32_t aw, uint32_t dstw, uint32_t pk, uint32_t cbank,
                   uint32_t dst, uint32_t ptr, uint32_t s0, uint32_t s1, uint32_t s2, uint32_t s3, int32_t imm) {
  Rec r;
  r.w0 = (op & 0xffu) | ((flags & 0xffu) << 8) | ((aw & 7u) << 16) | ((pk & 3u) << 19) | ((cbank & 31u) << 21) |
         ((dstw & 63u) << 26);
  r.w1 = (dst & 511u) | ((ptr & 511u) << 9) | ((s0 & 511u) << 18) | (((dstw >> 6) & 3u) << 27);
  r.w2 = (s1 & 511u) | ((s2 & 511u) << 9) | ((s3 & 511u) << 18);
  r.w3 = imm;
  return r;
}

// per-kernel descriptor (device)
struct KDesc {
  uint32_t first;       // global slot of instruction 0
  uint32_t n;           // instructions
  uint32_t param_base;  // R1 (bits 0..15); the kernel's GPR count (R38k) in bits 16..31
  uint32_t win0;        // first window id
};
GS_HD uint32_t kd_param_base(const KDesc& k) { return k.param_base & 0xffffu; }
GS_HD uint32_t kd_nregs(const KDesc& k) { return k.param_base >> 16; }

// per-window descriptor (device): windows never cross kernels
struct WDesc {
  uint32_t kernel, start, len, pad;
};

}  // namespace gs
