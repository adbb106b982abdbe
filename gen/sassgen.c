/* sassgen.c — deterministic synthetic SASS text generator (test / bench INPUT infrastructure).
 *
 * Writes sm_100 cuobjdump-syntax text (SURVEY [probe 2-3]) built from motifs shaped like the
 * paper's case-study kernels: naive-matmul inner loops, spills
 * (P:565-583), stencils, atomics, conversions, pointer chains
 * of exact length, and filler drawn from a real sm_100 opcode mix (SURVEY [probe 7]).
 * It contains none of the method's arithmetic; both the oracle and the GPU path consume its text.
 * Alongside the text it returns one class byte per instruction (gen/samples.py CLS_*), used only
 * to shape the synthetic stall-reason mix.
 */
#include <stdarg.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>

enum { CLS_ALU, CLS_MEM, CLS_CONSUMER, CLS_SMEM, CLS_BRA, CLS_BAR, CLS_OTHER };
enum { SH_GENERIC, SH_C1, SH_MIXBENCH, SH_JACOBI, SH_MATMUL, SH_CHAIN, SH_ATOMICS };

typedef struct {
  char *p, *end;
  int pc, n, ovf;
  uint8_t *cls;
  uint64_t s;
  int rr;          /* rotating register allocator */
  int loaded[8];   /* recently loaded registers (for consumers) */
  int nloaded;
} Em;

static uint64_t nx(Em *e) { /* splitmix64 */
  uint64_t z = (e->s += 0x9E3779B97F4A7C15ull);
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static int rnd(Em *e, int n) { return (int)(nx(e) % (uint64_t)n); }

static void ins(Em *e, int cls, const char *fmt, ...) {
  char body[160];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(body, sizeof body, fmt, ap);
  va_end(ap);
  int need = 64 + (int)strlen(body);
  if (e->p + need >= e->end) { e->ovf = 1; e->pc++; return; }
  e->p += sprintf(e->p, "        /*%04x*/                   %s ;\n", e->pc * 16, body);
  if (e->cls) e->cls[e->pc] = (uint8_t)cls;
  e->pc++;
}
/* registers: GPR R2..R199 (R0 = tid, R1 = stack pointer) */
static int reg1(Em *e) { e->rr = (e->rr + 1 + rnd(e, 5)) % 198; return 2 + e->rr; }
static int reg2(Em *e) { int r = reg1(e) & ~1; return r < 2 ? 2 : (r > 196 ? 196 : r); }
static int reg4(Em *e) { int r = reg1(e) & ~3; return r < 4 ? 4 : (r > 192 ? 192 : r); }
static void note_load(Em *e, int r) { e->loaded[e->nloaded++ % 8] = r; }
static int a_loaded(Em *e) { return e->nloaded ? e->loaded[rnd(e, e->nloaded < 8 ? e->nloaded : 8)] : reg1(e); }
static int param(Em *e) { return 0x380 + 8 * rnd(e, 8); }
static void offs(char *b, int off) {
  if (off > 0) sprintf(b, "+0x%x", off);
  else if (off < 0) sprintf(b, "+-0x%x", -off);
  else b[0] = 0;
}

static void prologue(Em *e) {
  ins(e, CLS_OTHER, "LDC R1, c[0x0][0x37c]");
  ins(e, CLS_OTHER, "S2R R0, SR_TID.X");
  ins(e, CLS_OTHER, "S2UR UR4, SR_CTAID.X");
  ins(e, CLS_OTHER, "LDCU.64 UR6, c[0x0][0x358]");
}

/* M7: one filler instruction from the sm_100 opcode mix ([probe 7]) */
static void filler(Em *e) {
  int c = rnd(e, 1000), d = reg1(e), a = reg1(e), b = reg1(e);
  if (c < 130) ins(e, CLS_ALU, "IMAD R%d, R%d, R%d, R%d", d, a, b, reg1(e));
  else if (c < 240) ins(e, CLS_ALU, "FMUL R%d, R%d, R%d", d, a, b);
  else if (c < 330) ins(e, CLS_CONSUMER, "FFMA R%d, R%d, R%d, R%d", d, a_loaded(e), b, d);
  else if (c < 400) ins(e, CLS_ALU, "ISETP.GE.AND P%d, PT, R%d, R%d, PT", rnd(e, 6), a, b);
  else if (c < 460) ins(e, CLS_ALU, "IADD3 R%d, PT, PT, R%d, 0x%x, RZ", d, a, 1 + rnd(e, 64));
  else if (c < 510) ins(e, CLS_ALU, "LOP3.LUT R%d, R%d, 0x%x, RZ, 0xc0, !PT", d, a, 1 + rnd(e, 255));
  else if (c < 560) ins(e, CLS_ALU, "SHF.L.U32 R%d, R%d, 0x%x, RZ", d, a, 1 + rnd(e, 8));
  else if (c < 610) ins(e, CLS_ALU, "MOV R%d, R%d", d, a);
  else if (c < 650) ins(e, CLS_ALU, "FADD R%d, R%d, R%d", d, a, b);
  else if (c < 710) {
    int q = reg4(e), x = reg4(e), y = reg4(e);
    ins(e, CLS_ALU, "HMMA.16816.F32 R%d, R%d, R%d, R%d", q, x, y, q);
  } else if (c < 750) ins(e, CLS_SMEM, "LDSM.16.M88.4 R%d, [R%d+UR4]", reg4(e), a);
  else if (c < 775) { ins(e, CLS_SMEM, "LDS R%d, [R%d+UR4+0x%x]", d, a, 4 * rnd(e, 64)); note_load(e, d); }
  else if (c < 790) ins(e, CLS_SMEM, "STS [R%d+UR4], R%d", a, b);
  else if (c < 804) ins(e, CLS_MEM, "LDGSTS.E.BYPASS.128 [R%d+UR4], desc[UR6][R%d.64]", a, reg2(e));
  else if (c < 814) { int r = reg2(e); ins(e, CLS_MEM, "LDG.E.128 R%d, desc[UR6][R%d.64+0x%x]", reg4(e), r, 16 * rnd(e, 4)); }
  else if (c < 818) { int r = reg2(e); ins(e, CLS_MEM, "LDG.E.CONSTANT R%d, desc[UR6][R%d.64]", d, r); note_load(e, d); }
  else if (c < 838) ins(e, CLS_ALU, "I2FP.F32.S32 R%d, R%d", d, a);
  else if (c < 848) ins(e, CLS_ALU, "F2FP.BF16.F32.PACK_AB R%d, R%d, R%d", d, a, b);
  else if (c < 860) ins(e, CLS_ALU, "ISETP.NE.U32.AND P%d, PT, R%d, RZ, PT", rnd(e, 6), a);
  else if (c < 868) { int r = reg2(e); ins(e, CLS_MEM, "STG.E desc[UR6][R%d.64+0x%x], R%d", r, 4 * rnd(e, 8), a); }
  else if (c < 876) ins(e, CLS_BAR, "BAR.SYNC.DEFER_BLOCKING 0x0");
  else if (c < 900) ins(e, CLS_ALU, "IMAD.MOV.U32 R%d, RZ, RZ, R%d", d, a);
  else if (c < 920) ins(e, CLS_ALU, "IMAD.WIDE R%d, R%d, 0x4, R%d", reg2(e), a, reg2(e));
  else if (c < 940) ins(e, CLS_ALU, "LEA R%d, P%d, R%d, UR%d, 0x2", d, rnd(e, 6), a, 8 + 2 * rnd(e, 8));
  else if (c < 960) ins(e, CLS_ALU, "VIADD R%d, R%d, 0x%x", d, a, 1 + rnd(e, 32));
  else if (c < 975) ins(e, CLS_ALU, "FMNMX R%d, R%d, R%d, !PT", d, a, b);
  else if (c < 990) ins(e, CLS_ALU, "MUFU.EX2 R%d, R%d", d, a);
  else ins(e, CLS_ALU, "SEL R%d, R%d, R%d, P%d", d, a, b, rnd(e, 6));
}

/* M1: naive-matmul inner loop, unroll u (A: u contiguous 32-bit loads off one base; B: strided) */
static void m_matmul(Em *e, int u) {
  int pa = param(e), pb = param(e);
  int ra = reg2(e), rb = reg2(e), ri = reg1(e), rj = reg1(e), acc = reg1(e), cnt = reg1(e);
  ins(e, CLS_OTHER, "LDCU.64 UR8, c[0x0][0x%x]", pa);
  ins(e, CLS_OTHER, "LDC.64 R%d, c[0x0][0x%x]", rb, pb);
  ins(e, CLS_ALU, "MOV R%d, UR8", ra);
  ins(e, CLS_ALU, "MOV R%d, UR9", ra + 1);
  ins(e, CLS_ALU, "IMAD.WIDE R%d, R%d, 0x4, R%d", ra, ri, ra);
  int top = e->pc;
  int va[16], vb[16];
  char o[32];
  for (int k = 0; k < u; k++) {
    va[k] = reg1(e);
    offs(o, 4 * k - 4 * (u / 2));
    ins(e, CLS_MEM, "LDG.E R%d, desc[UR6][R%d.64%s]", va[k], ra, o);
  }
  int cur = rb;
  for (int k = 0; k < u; k++) {
    int nb = reg2(e);
    ins(e, CLS_ALU, "IMAD.WIDE R%d, R%d, 0x4, R%d", nb, k ? rj : ri, cur);
    vb[k] = reg1(e);
    ins(e, CLS_MEM, "LDG.E R%d, desc[UR6][R%d.64]", vb[k], nb);
    cur = nb;
  }
  for (int k = 0; k < u; k++) ins(e, CLS_CONSUMER, "FFMA R%d, R%d, R%d, R%d", acc, va[k], vb[k], acc);
  ins(e, CLS_ALU, "IADD3 R%d, PT, PT, R%d, 0x%x, RZ", cnt, cnt, u);
  ins(e, CLS_ALU, "ISETP.NE.AND P1, PT, R%d, RZ, PT", cnt);
  ins(e, CLS_BRA, "@P1 BRA 0x%x", top * 16);
  note_load(e, acc);
}

/* M2: spill — producer then STL, later LDL.LU then consumer */
static void m_spill(Em *e, int wide) {
  int x = wide ? reg2(e) : reg1(e), off = 4 * rnd(e, 64) * (wide ? 2 : 1);
  if (wide) ins(e, CLS_ALU, "IMAD.WIDE R%d, R%d, 0x4, R%d", x, reg1(e), reg2(e));
  else if (rnd(e, 2)) ins(e, CLS_ALU, "IADD3 R%d, PT, PT, R%d, R%d, RZ", x, reg1(e), reg1(e));
  else ins(e, CLS_CONSUMER, "FFMA R%d, R%d, R%d, R%d", x, a_loaded(e), reg1(e), reg1(e));
  ins(e, CLS_MEM, wide ? "STL.64 [R1+0x%x], R%d" : "STL [R1+0x%x], R%d", off, x);
  filler(e);
  ins(e, CLS_MEM, wide ? "LDL.LU.64 R%d, [R1+0x%x]" : "LDL R%d, [R1+0x%x]", x, off);
  ins(e, CLS_CONSUMER, "FFMA R%d, R%d, R%d, R%d", reg1(e), x, reg1(e), reg1(e));
}

/* M3: stencil — up to 5 loads around one base (+-4 and +row), store to another param */
static void m_stencil(Em *e) {
  int pi = param(e), po = param(e);
  while (po == pi) po = param(e);
  int rp = reg2(e), rq = reg2(e), rr = reg2(e), ri = reg1(e), rn = reg1(e), v[5];
  ins(e, CLS_OTHER, "LDC.64 R%d, c[0x0][0x%x]", rp, pi);
  ins(e, CLS_ALU, "IMAD.WIDE R%d, R%d, 0x4, R%d", rq, ri, rp);
  ins(e, CLS_ALU, "IMAD.WIDE R%d, R%d, 0x4, R%d", rr, rn, rq);
  for (int k = 0; k < 5; k++) v[k] = reg1(e);
  ins(e, CLS_MEM, "LDG.E R%d, desc[UR6][R%d.64+-0x4]", v[0], rq);
  ins(e, CLS_MEM, "LDG.E R%d, desc[UR6][R%d.64]", v[1], rq);
  ins(e, CLS_MEM, "LDG.E R%d, desc[UR6][R%d.64+0x4]", v[2], rq);
  ins(e, CLS_MEM, "LDG.E R%d, desc[UR6][R%d.64]", v[3], rr);
  ins(e, CLS_CONSUMER, "FADD R%d, R%d, R%d", v[4], v[0], v[2]);
  ins(e, CLS_CONSUMER, "FADD R%d, R%d, R%d", v[4], v[4], v[3]);
  ins(e, CLS_CONSUMER, "FFMA R%d, R%d, -4, R%d", v[4], v[1], v[4]);
  int rs = reg2(e), rt = reg2(e);
  ins(e, CLS_OTHER, "LDC.64 R%d, c[0x0][0x%x]", rs, po);
  ins(e, CLS_ALU, "IMAD.WIDE R%d, R%d, 0x4, R%d", rt, ri, rs);
  ins(e, CLS_MEM, "STG.E desc[UR6][R%d.64], R%d", rt, v[4]);
}

/* M4: shared + global atomics in a loop */
static void m_atomics(Em *e) {
  int k = reg1(e), lo = reg2(e), v = reg1(e), top;
  ins(e, CLS_ALU, "LEA R%d, R%d, UR4, 0x2", k, reg1(e));
  ins(e, CLS_OTHER, "LDCU.64 UR10, c[0x0][0x%x]", param(e));
  top = e->pc;
  ins(e, CLS_SMEM, "ATOMS.POPC.INC.32 RZ, [R%d+UR4]", k);
  ins(e, CLS_ALU, "IADD3 R%d, P0, PT, R%d, UR10, RZ", lo, reg1(e));
  ins(e, CLS_ALU, "IMAD.X R%d, RZ, RZ, UR11, P0", lo + 1);
  ins(e, CLS_MEM, "REDG.E.ADD.STRONG.GPU desc[UR6][R%d.64], R%d", lo, v);
  ins(e, CLS_ALU, "ISETP.GE.AND P0, PT, R%d, UR5, PT", reg1(e));
  ins(e, CLS_BRA, "@!P0 BRA 0x%x", top * 16);
}

/* M5: conversions */
static void m_conv(Em *e) {
  ins(e, CLS_ALU, "I2FP.F32.S32 R%d, R%d", reg1(e), reg1(e));
  ins(e, CLS_ALU, "F2F.F32.F64 R%d, R%d", reg1(e), reg2(e));
}

/* M6: pointer chain needing exactly L+1 last-writer steps (L ALU links + the LDC.64 root) */
static void m_chain(Em *e, int L) {
  int r = reg2(e);
  ins(e, CLS_OTHER, "LDC.64 R%d, c[0x0][0x%x]", r, param(e));
  for (int k = 0; k < L; k++) {
    int nr = 2 + ((r - 2 + 2 + 2 * rnd(e, 4)) % 190);
    nr &= ~1;
    if (nr == r) nr = (r + 2 > 190) ? 2 : r + 2;
    switch (k % 3) {
      case 0: ins(e, CLS_ALU, "IADD3 R%d, P0, PT, R%d, 0x10, RZ", nr, r); break;
      case 1: ins(e, CLS_ALU, "MOV R%d, R%d", nr, r); break;
      default: ins(e, CLS_ALU, "IMAD.WIDE R%d, R%d, 0x4, R%d", nr, 0, r); break;
    }
    r = nr;
  }
  int v = reg1(e);
  ins(e, CLS_MEM, "LDG.E R%d, desc[UR6][R%d.64]", v, r);
  ins(e, CLS_CONSUMER, "FADD R%d, R%d, R%d", reg1(e), v, v);
}

/* mixbench-shaped block: 8 contiguous loads (SP) or 8 LDG.E.64 (DP), MAD loop, store */
static void m_mixbench(Em *e, int dp) {
  int rb = reg2(e), v[8], top, cnt = reg1(e);
  ins(e, CLS_OTHER, "LDC.64 R%d, c[0x0][0x%x]", rb, param(e));
  ins(e, CLS_ALU, "IMAD.WIDE R%d, R%d, 0x%x, R%d", rb, reg1(e), dp ? 8 : 4, rb);
  for (int k = 0; k < 8; k++) {
    v[k] = dp ? reg2(e) : reg1(e);
    ins(e, CLS_MEM, dp ? "LDG.E.64 R%d, desc[UR6][R%d.64+0x%x]" : "LDG.E R%d, desc[UR6][R%d.64+0x%x]",
        v[k], rb, k * (dp ? 8 : 4));
  }
  ins(e, CLS_OTHER, "LDCU%s UR8, c[0x0][0x380]", dp ? ".64" : "");
  top = e->pc;
  for (int k = 0; k < 8; k++)
    ins(e, CLS_CONSUMER, dp ? "DFMA R%d, R%d, R%d, UR8" : "FFMA R%d, R%d, R%d, UR8", v[k], v[k], v[k]);
  ins(e, CLS_ALU, "IADD3 R%d, PT, PT, R%d, 0x1, RZ", cnt, cnt);
  ins(e, CLS_ALU, "ISETP.NE.AND P1, PT, R%d, RZ, PT", cnt);
  ins(e, CLS_BRA, "@P1 BRA 0x%x", top * 16);
  ins(e, CLS_MEM, dp ? "STG.E.64 desc[UR6][R%d.64], R%d" : "STG.E desc[UR6][R%d.64], R%d", rb, v[0]);
}

static int motif_size_max = 72;

static void body(Em *e, int shape, int arg, int n) {
  /* shape-specific leading motifs */
  switch (shape) {
    case SH_C1:
      m_matmul(e, 8);
      for (int k = 0; k < 12; k++) m_spill(e, k % 4 == 3);  /* 12 STL + 12 LDL */
      m_stencil(e);
      break;
    case SH_MIXBENCH:
      while (e->pc < n * 3 / 10) m_mixbench(e, 0);
      while (e->pc < n * 6 / 10) m_mixbench(e, 1);
      break;
    case SH_JACOBI:
      while (e->pc < n * 6 / 10) { m_stencil(e); for (int k = 0; k < 6; k++) ins(e, CLS_ALU, "I2FP.F32.S32 R%d, R%d", reg1(e), reg1(e)); }
      break;
    case SH_MATMUL:
      while (e->pc < n * 6 / 10) m_matmul(e, 8);
      break;
    case SH_CHAIN:
      m_chain(e, arg);
      break;
    case SH_ATOMICS:
      while (e->pc < n * 5 / 10) m_atomics(e);
      break;
    default:
      break;
  }
  /* generic motif mix (C3 rates) then single fillers to the exact size */
  while (n - 2 - e->pc > motif_size_max) {
    /* per-step motif odds (of 10000) tuned to the C3 rates: LDG ~1.6%, STG ~0.8%, LDS ~2.5%,
       conversions ~3%, STL/LDL ~0.2%, global atomics ~0.05% */
    int c = rnd(e, 10000);
    if (shape != SH_GENERIC || c < 9912) filler(e);
    else if (c < 9930) m_matmul(e, 2 + 2 * rnd(e, 4));
    else if (c < 9945) m_stencil(e);
    else if (c < 9955) m_spill(e, rnd(e, 4) == 0);
    else if (c < 9960) m_atomics(e);
    else if (c < 9990) m_conv(e);
    else m_chain(e, 2 + rnd(e, 12));
  }
  while (e->pc < n - 2) filler(e);
}

/* Generates n_kernels kernels into buf. Returns bytes written, or -1 if cap is too small.
 * cls (optional) receives one class byte per instruction, concatenated over kernels.
 * shapes/args/sizes: per kernel. names: printed as "Function : <prefix><k>". */
int64_t gsgen_kernels(char *buf, int64_t cap, int n_kernels, const int32_t *shapes, const int32_t *args,
                      const int32_t *sizes, uint64_t seed, uint8_t *cls, const char *prefix) {
  char *p = buf, *end = buf + cap;
  int64_t slot = 0;
  if (end - p < 64) return -1;
  p += sprintf(p, "\n\tcode for sm_100a\n\t.target\tsm_100a\n\n");
  for (int k = 0; k < n_kernels; k++) {
    if (end - p < 256) return -1;
    p += sprintf(p, "\t\tFunction : %s%d\n\t.headerflags\t@\"EF_CUDA_SM100 EF_CUDA_VIRTUAL_SM(EF_CUDA_SM100)\"\n",
                 prefix, k);
    Em e;
    memset(&e, 0, sizeof e);
    e.p = p; e.end = end; e.cls = cls ? cls + slot : NULL;
    e.s = seed * 0x100000001B3ull + (uint64_t)k * 0x9E3779B97F4A7C15ull + 12345;
    int n = sizes[k] < 8 ? 8 : sizes[k];
    prologue(&e);
    body(&e, shapes[k], args ? args[k] : 0, n);
    ins(&e, CLS_OTHER, "EXIT");
    ins(&e, CLS_BRA, "BRA 0x%x", e.pc * 16);
    if (e.ovf) return -1;
    if (e.pc != n) return -2;
    p = e.p;
    if (end - p < 32) return -1;
    p += sprintf(p, "\t\t..........\n\n\n");
    slot += n;
  }
  return p - buf;
}
