// loader.cpp — SASS text -> packed 16-byte records (§2.1).
//
// Product code (host side of gs_load_sass). Written independently of oracle/gs_oracle.cpp from the
// readings in DESIGN.md §3 (R1, R2, R6, R7, R23-R28, R33). Kernels are parsed in parallel: a first
// sequential pass only finds kernel headers (cuobjdump "Function : f", nvdisasm ".text.f:") and
// arch lines; each kernel's lines are then tokenised by a worker thread into records. nvdisasm
// branch targets are labels (BRA `(.L_x_3)); a label names the pc of the next instruction, and
// only backward targets matter (R13), so a label is resolved when its branch is reached.
#include <algorithm>
#include <atomic>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <string>
#include <string_view>
#include <unordered_map>
#include <thread>
#include <utility>
#include <vector>

#include "loader.h"

namespace gs {
namespace {

struct Sv {  // non-owning text span
  const char* p = nullptr;
  size_t n = 0;
  template <size_t N>  // literals: length known at compile time (the parser compares thousands per line)
  bool eq(const char (&s)[N]) const { return n == N - 1 && memcmp(p, s, N - 1) == 0; }
  bool eqz(const char* s) const { size_t m = strlen(s); return m == n && memcmp(p, s, n) == 0; }
  char operator[](size_t i) const { return p[i]; }
};

inline bool is_ws(char c) { return c == ' ' || c == '\t' || c == '\r' || c == '\n'; }
inline Sv trim(Sv s) {
  while (s.n && is_ws(s.p[0])) { s.p++; s.n--; }
  while (s.n && is_ws(s.p[s.n - 1])) s.n--;
  return s;
}
inline bool contains(Sv s, const char* needle, size_t* at = nullptr) {
  const size_t m = strlen(needle);
  if (m > s.n) return false;
  const void* f = memmem(s.p, s.n, needle, m);
  if (!f) return false;
  if (at) *at = (size_t)((const char*)f - s.p);
  return true;
}
template <size_t N>
inline bool starts(Sv s, const char (&pre)[N]) { return s.n >= N - 1 && memcmp(s.p, pre, N - 1) == 0; }
inline int hexv(char c) {
  if (c >= '0' && c <= '9') return c - '0';
  if (c >= 'a' && c <= 'f') return c - 'a' + 10;
  if (c >= 'A' && c <= 'F') return c - 'A' + 10;
  return -1;
}

// integer literal: optional sign, then 0x-hex or decimal, nothing else
bool to_int(Sv s, long long* v) {
  s = trim(s);
  bool neg = false;
  if (s.n && (s[0] == '-' || s[0] == '+')) { neg = s[0] == '-'; s.p++; s.n--; }
  if (!s.n) return false;
  long long x = 0;
  if (s.n > 2 && s[0] == '0' && (s[1] == 'x' || s[1] == 'X')) {
    for (size_t i = 2; i < s.n; i++) { int h = hexv(s[i]); if (h < 0) return false; x = x * 16 + h; }
  } else {
    for (size_t i = 0; i < s.n; i++) { if (s[i] < '0' || s[i] > '9') return false; x = x * 10 + (s[i] - '0'); }
  }
  *v = neg ? -x : x;
  return true;
}

Sv unprefix(Sv s) {
  while (s.n && (s[0] == '-' || s[0] == '!' || s[0] == '~' || s[0] == '|')) { s.p++; s.n--; }
  return s;
}

// register token -> id (R6): Rn (n<=254) RZ URn (n<=62) URZ; suffix from the first '.' ignored
int reg_id(Sv s) {
  size_t cut = s.n;
  for (size_t i = 0; i < s.n; i++) if (s[i] == '.') { cut = i; break; }
  s.n = cut;
  while (s.n && s[s.n - 1] == '|') s.n--;
  bool ur = false;
  size_t i = 0;
  if (s.n >= 2 && s[0] == 'U' && s[1] == 'R') { ur = true; i = 2; }
  else if (s.n >= 1 && s[0] == 'R') i = 1;
  else return -1;
  size_t m = s.n - i;
  if (m == 1 && s[i] == 'Z') return ur ? kURZ : kRZ;
  if (m == 0 || m > 3) return -1;
  int v = 0;
  for (size_t q = i; q < s.n; q++) { if (s[q] < '0' || s[q] > '9') return -1; v = v * 10 + (s[q] - '0'); }
  if (ur) return v <= 62 ? 256 + v : -1;
  return v <= 254 ? v : -1;
}

bool is_pred(Sv s) {
  size_t i;
  if (s.n >= 2 && s[0] == 'U' && s[1] == 'P') i = 2;
  else if (s.n >= 1 && s[0] == 'P') i = 1;
  else return false;
  return s.n == i + 1 && (s[i] == 'T' || (s[i] >= '0' && s[i] <= '7'));
}

enum Kind { T_REG, T_PRED, T_CREF, T_MEM, T_MISC };
struct Operand {
  Kind k = T_MISC;
  int reg = -1;              // T_REG
  int bank = 0;              // T_CREF
  long long imm = 0;         // T_CREF offset, T_MEM offset
  int base = -1;             // T_MEM base register
  int regs[8];               // all registers inside (brackets too), in order
  int nregs = 0;
  bool wide = false;         // T_MEM: base written Rb.64
  bool predvar = false;      // T_PRED: a real predicate (not PT / UPT)
  void add(int r) { if (nregs < 8) regs[nregs++] = r; }
};

// bracket body "R4.64+-0x10": registers (first one = base if wanted) and immediate sum
void scan_bracket(Sv b, Operand* o, bool want_base, long long* sum) {
  size_t s = 0;
  while (s <= b.n) {
    size_t e = s;
    while (e < b.n && b[e] != '+') e++;
    Sv term = trim(Sv{b.p + s, e - s});
    if (term.n) {
      int r = reg_id(unprefix(term));
      long long v;
      if (r >= 0) {
        o->add(r);
        if (want_base && o->base < 0) o->base = r;
      } else if (to_int(term, &v)) {
        *sum += v;
      }
    }
    s = e + 1;
  }
}

Operand classify(Sv raw) {
  Operand o;
  Sv t = trim(raw);
  Sv u = unprefix(t);
  if (u.n > 2 && u[0] == 'c' && u[1] == '[') {
    o.k = T_CREF;
    size_t a = 2;
    while (a < u.n && u[a] != ']') a++;
    long long bank = 0;
    to_int(Sv{u.p + 2, a - 2}, &bank);
    o.bank = (int)bank;
    size_t b0 = a;
    while (b0 < u.n && u[b0] != '[') b0++;
    if (b0 < u.n) {
      size_t b1 = b0;
      while (b1 < u.n && u[b1] != ']') b1++;
      if (b1 < u.n) scan_bracket(Sv{u.p + b0 + 1, b1 - b0 - 1}, &o, false, &o.imm);
    }
    return o;
  }
  size_t lb = u.n;
  for (size_t i = 0; i < u.n; i++) if (u[i] == '[') { lb = i; }
  if (lb < u.n) {  // memory operand; lb = last '['
    o.k = T_MEM;
    size_t i = 0;
    while (i < u.n) {
      if (u[i] != '[') { i++; continue; }
      size_t c = i;
      while (c < u.n && u[c] != ']') c++;
      long long dummy = 0;
      if (i == lb) {
        scan_bracket(Sv{u.p + i + 1, c - i - 1}, &o, true, &o.imm);
        o.wide = contains(Sv{u.p + i + 1, c - i - 1}, ".64");
      }
      else scan_bracket(Sv{u.p + i + 1, c - i - 1}, &o, false, &dummy);
      i = c + 1;
    }
    return o;
  }
  int r = reg_id(u);
  if (r >= 0) { o.k = T_REG; o.reg = r; o.add(r); return o; }
  if (is_pred(u)) {
    o.k = T_PRED;
    o.predvar = u[u.n - 1] != 'T';
    return o;
  }
  o.k = T_MISC;  // immediates, floats, SR_*, B0, PR, ...
  return o;
}

struct OpName { const char* s; uint8_t id; };
const OpName kOps[] = {
    {"LDG", OP_LDG}, {"LDL", OP_LDL}, {"STL", OP_STL}, {"STG", OP_STG}, {"ST", OP_ST}, {"LD", OP_LD},
    {"LDS", OP_LDS}, {"STS", OP_STS}, {"LDSM", OP_LDSM}, {"ATOM", OP_ATOM}, {"ATOMG", OP_ATOMG},
    {"ATOMS", OP_ATOMS}, {"RED", OP_RED}, {"REDG", OP_REDG}, {"SUST", OP_SUST}, {"SULD", OP_SULD},
    {"SUATOM", OP_SUATOM}, {"TLD", OP_TLD}, {"TLD4", OP_TLD4}, {"TLDS", OP_TLDS}, {"TEX", OP_TEX},
    {"TMML", OP_TMML}, {"TXD", OP_TXD}, {"TXQ", OP_TXQ}, {"LDTM", OP_LDTM}, {"LDC", OP_LDC},
    {"LDCU", OP_LDCU}, {"ULDC", OP_ULDC}, {"S2R", OP_S2R}, {"S2UR", OP_S2UR}, {"CS2R", OP_CS2R},
    {"BRA", OP_BRA}, {"F2F", OP_F2F}, {"F2I", OP_F2I}, {"I2F", OP_I2F}, {"I2I", OP_I2I},
    {"I2FP", OP_I2FP}, {"F2IP", OP_F2IP}, {"F2FP", OP_F2FP}, {"FADD", OP_FADD}, {"FMUL", OP_FMUL},
    {"FFMA", OP_FFMA}, {"FMNMX", OP_FMNMX}, {"DADD", OP_DADD}, {"DMUL", OP_DMUL}, {"DFMA", OP_DFMA},
    {"HADD2", OP_HADD2}, {"HMUL2", OP_HMUL2}, {"HFMA2", OP_HFMA2}, {"MUFU", OP_MUFU},
    {"IADD3", OP_IADD3}, {"VIADD", OP_VIADD}, {"IMAD", OP_IMAD}, {"IMUL", OP_IMUL},
    {"IMNMX", OP_IMNMX}, {"VIMNMX", OP_VIMNMX}, {"IABS", OP_IABS}, {"LEA", OP_LEA},
    {"ULEA", OP_ULEA}, {"UIADD3", OP_UIADD3}, {"UIMAD", OP_UIMAD}, {"HMMA", OP_HMMA},
    {"DMNMX", OP_DMNMX}, {"FCHK", OP_FCHK}, {"CALL", OP_CALL}, {"RET", OP_RET}, {"BRX", OP_BRX},
};

uint8_t op_lookup(Sv m) {
  static const std::unordered_map<std::string_view, uint8_t> tab = [] {
    std::unordered_map<std::string_view, uint8_t> t;
    for (const auto& o : kOps) t.emplace(o.s, o.id);
    return t;
  }();
  const auto it = tab.find(std::string_view(m.p, m.n));
  return it == tab.end() ? (uint8_t)OP_OTHER : it->second;
}

struct Line {
  const char* p;
  size_t n;
  long lineno;
};

// Register-pressure inputs of one instruction (O16 / R36, R38): GPR uses with operand widths
// expanded, guard, exit, predicate/register condition of a branch, branch target (pc) or unresolved
// label, indirect-branch target labels, highest GPR touched.
struct LiveOut {
  std::vector<uint8_t>* uses = nullptr;
  bool guarded = false, exit = false, brpred = false;
  long long target = -1;
  std::string label;
  std::vector<std::string> brx;  // nvdisasm BRANCH_TARGETS of a BRX (R38i)
  int maxreg = -1;
};

inline bool is64type(Sv m) { return m.eq("F64") || m.eq("S64") || m.eq("U64"); }
inline bool isinttype(Sv m) {
  static const char* k[] = {"S64", "U64", "S32", "U32", "S16", "U16", "S8", "U8"};
  for (auto* x : k) if (m.eqz(x)) return true;
  return false;
}
inline bool isfloattype(Sv m) {
  static const char* k[] = {"F64", "F32", "F16", "BF16", "TF32", "E4M3", "E5M2"};
  for (auto* x : k) if (m.eqz(x)) return true;
  return false;
}

// R38e: register widths {destination, source} of a conversion from the roles of its type modifiers
void conv_roles(Sv mn, const Sv* mods, int nm, uint32_t* dw, uint32_t* sw) {
  Sv t[8];
  int nt = 0;
  for (int q = 0; q < nm && nt < 8; q++)
    if (isinttype(mods[q]) || isfloattype(mods[q])) t[nt++] = mods[q];
  Sv d{}, src{};
  if (mn.eq("F2F") || mn.eq("I2I") || mn.eq("F2FP")) {
    if (nt >= 1) d = t[0];
    if (nt >= 2) src = t[1];
  } else if (mn.eq("I2F") || mn.eq("I2FP")) {
    for (int q = 0; q < nt; q++) (isfloattype(t[q]) ? d : src) = t[q];
  } else if (mn.eq("F2I") || mn.eq("F2IP")) {
    for (int q = 0; q < nt; q++) (isinttype(t[q]) ? d : src) = t[q];
  }
  *dw = d.n && is64type(d) ? 2 : 1;
  *sw = src.n && is64type(src) ? 2 : 1;
}

// R38d: registers per thread of a tensor-memory access LDTM/STTM[.<shape>].x<N>
uint32_t tmem_width(const Sv* mods, int nm) {
  uint32_t per = 1, x = 1;
  for (int q = 0; q < nm; q++) {
    if (mods[q].eq("16dp128bit")) per = 2;
    else if (mods[q].eq("16dp256bit")) per = 4;
    else if (mods[q].n > 1 && mods[q][0] == 'x' && mods[q][1] >= '0' && mods[q][1] <= '9') {
      x = 0;
      for (size_t k = 1; k < mods[q].n && mods[q][k] >= '0' && mods[q][k] <= '9'; k++) x = x * 10 + (mods[q][k] - '0');
    }
  }
  return per * x;
}

// One instruction -> record. Returns false with msg on a malformed line.
bool pack_line(Sv body, long lineno, size_t index, Rec* out, std::string* msg, LiveOut* lo) {
  body = trim(body);
  if (body.n && body[0] == '@') {  // guard predicate
    lo->guarded = !starts(body, "@PT") && !starts(body, "@UPT");
    size_t i = 0;
    while (i < body.n && !is_ws(body[i])) i++;
    body = trim(Sv{body.p + i, body.n - i});
  }
  size_t i = 0;
  while (i < body.n && !is_ws(body[i])) i++;
  Sv opc{body.p, i};
  Sv rest = trim(Sv{body.p + i, body.n - i});
  // mnemonic and modifiers
  Sv mods[16];
  int nm = 0;
  size_t d = 0;
  while (d < opc.n && opc[d] != '.') d++;
  Sv mn{opc.p, d};
  while (d < opc.n && nm < 16) {
    size_t e = d + 1;
    while (e < opc.n && opc[e] != '.') e++;
    mods[nm++] = Sv{opc.p + d + 1, e - d - 1};
    d = e;
  }
  auto has = [&](const auto& m) { for (int q = 0; q < nm; q++) if (mods[q].eq(m)) return true; return false; };
  uint32_t op = op_lookup(mn);
  if (op == OP_IMAD && nm > 0 && mods[0].eq("MOV")) op = OP_IMAD_MOV;
  // operands: top-level commas
  Operand ops[16];
  Sv raw_last;
  int no = 0;
  {
    // operands are separated by top-level commas, or by blanks where SASS writes no comma
    // ("RET.REL.NODEC R2 0x0", "BRX R4 -0x43d0", R38i)
    int depth = 0;
    size_t s = 0;
    for (size_t q = 0; q <= rest.n; q++) {
      char c = q < rest.n ? rest[q] : ',';
      if (c == '[' || c == '{') depth++;
      else if (c == ']' || c == '}') depth--;
      const bool blank = (c == ' ' || c == '\t') && depth == 0;
      if ((c == ',' && depth == 0) || q == rest.n || blank) {
        Sv tok{rest.p + s, q - s};
        if (blank && !trim(tok).n) { s = q + 1; continue; }
        if (q < rest.n || trim(tok).n) {
          if (no >= 16) { *msg = "too many operands"; return false; }
          ops[no++] = classify(tok);
          raw_last = tok;
        }
        s = q + 1;
      }
    }
  }
  // HMMA fragment widths (R38c): m16 n8 kK tile, input element bits b -> A = 16Kb/1024, B = 8Kb/1024
  // registers, accumulator 4 (F32) or 2 (F16)
  uint32_t mma_a = 1, mma_b = 1, mma_acc = 1;
  if (op == OP_HMMA) {
    uint32_t K = 8, bits = 16;
    bool acc_seen = false, acc16 = false;
    for (int q = 0; q < nm; q++) {
      if (q == 0 && mods[q].n >= 4 && mods[q][0] >= '0' && mods[q][0] <= '9') {
        K = 0;
        for (size_t k = 3; k < mods[q].n; k++) K = K * 10 + (uint32_t)(mods[q][k] - '0');
      } else if (!acc_seen && isfloattype(mods[q])) {
        acc_seen = true;
        acc16 = mods[q].eq("F16");
      } else if (mods[q].eq("TF32")) bits = 32;
      else if (mods[q].eq("E4M3") || mods[q].eq("E5M2")) bits = 8;
    }
    mma_a = std::max(1u, 16 * K * bits / 1024);
    mma_b = std::max(1u, 8 * K * bits / 1024);
    mma_acc = acc16 ? 2 : 4;
  }
  uint32_t cdw = 1, csw = 1;
  const bool conv = op == OP_F2F || op == OP_I2F || op == OP_F2I || op == OP_I2I || op == OP_I2FP ||
                    op == OP_F2IP || op == OP_F2FP;
  if (conv) conv_roles(mn, mods, nm, &cdw, &csw);
  // destination (R23); opcodes whose register operands are all read have none (R38f)
  const bool no_dst = mn.eq("WARPSYNC") || mn.eq("BRX") || mn.eq("BRXU") || mn.eq("JMX") || mn.eq("JMXU") ||
                      mn.eq("RET") || mn.eq("CALL") || mn.eq("NANOSLEEP") || mn.eq("BAR") || mn.eq("YIELD") ||
                      mn.eq("BPT");
  int dpos = -1, dpos2 = -1;
  if (no_dst) dpos = -1;
  else if (no >= 1 && ops[0].k == T_REG) dpos = 0;
  else if (no >= 2 && ops[0].k == T_PRED && ops[1].k == T_REG && op != OP_FCHK) dpos = 1;
  uint32_t dst = kRegNone, dstw = 0, dst2 = kRegNone;
  if (dpos >= 0) {
    dst = (uint32_t)ops[dpos].reg;
    // width table W (R24 as revised by R38)
    if (has("256")) dstw = 4;  // R38a: each of the two destination quads
    else if (has("128")) dstw = 4;
    else if (op == OP_HMMA) dstw = mma_acc;
    else if (mn.eq("LDSM")) dstw = has("4") ? 4 : (has("2") ? 2 : 1);
    else if (op == OP_LDTM) dstw = tmem_width(mods, nm);
    else if (has("64") || has("WIDE")) dstw = 2;
    else if (op == OP_CS2R) dstw = has("32") ? 1 : 2;  // R38b
    else if (mn.eq("LEPC")) dstw = 2;
    else if (op == OP_DADD || op == OP_DMUL || op == OP_DFMA || op == OP_DMNMX) dstw = 2;
    else if (conv) dstw = cdw;
    else dstw = 1;
    if (dstw > 255) { *msg = "destination wider than 255 registers"; return false; }
    if (has("256") && dpos + 1 < no && ops[dpos + 1].k == T_REG) {  // R38a: LDG.E.ENL2.256 Ra, Rb
      dpos2 = dpos + 1;
      dst2 = (uint32_t)ops[dpos2].reg;
    }
  }
  const int last_dst = dpos2 >= 0 ? dpos2 : dpos;
  // memory operand
  int mem = -1;
  for (int q = 0; q < no; q++) if (ops[q].k == T_MEM) { mem = q; break; }
  uint32_t flags = 0, aw = AW_NONE, s[4] = {kRegNone, kRegNone, kRegNone, kRegNone};
  int32_t imm = 0;
  uint32_t cbank = 0;
  if (has("CONSTANT")) flags |= F_CONSTANT;
  uint32_t cls = op_class(op);
  if (mem >= 0) {
    flags |= F_HASMEM;
    const Operand& m = ops[mem];
    s[0] = m.base >= 0 ? (uint32_t)m.base : kRegNone;
    imm = (int32_t)m.imm;
    for (int q = mem + 1; q < no; q++)
      if (ops[q].k == T_REG) { s[1] = (uint32_t)ops[q].reg; break; }
    aw = AW_32;
    for (int q = 0; q < nm; q++) {
      if (mods[q].eq("U8") || mods[q].eq("S8")) { aw = AW_8; break; }
      if (mods[q].eq("U16") || mods[q].eq("S16")) { aw = AW_16; break; }
      if (mods[q].eq("64")) { aw = AW_64; break; }
      if (mods[q].eq("128")) { aw = AW_128; break; }
      if (mods[q].eq("256")) { aw = AW_256; break; }
    }
  }
  if (dst2 != kRegNone) {  // the second quad travels in s2 (record.h)
    s[2] = dst2;
    flags |= F_DST2;
  }
  if (cls & C_ARITH) {  // register sources after dst (R25), at most 4
    int ns = 0;
    for (int q = last_dst + 1; q < no; q++)
      for (int t = 0; t < ops[q].nregs; t++) {
        int r = ops[q].regs[t];
        if (!reg_live((uint32_t)r)) continue;
        if (ns == 4) { *msg = "arithmetic instruction with more than 4 register sources"; return false; }
        s[ns++] = (uint32_t)r;
      }
  }
  // constant-bank load (trace terminal): c[bank][off]
  if (cls & C_CONSTLOAD) {
    for (int q = dpos + 1; q < no; q++)
      if (ops[q].k == T_CREF) { cbank = (uint32_t)ops[q].bank; imm = (int32_t)ops[q].imm; break; }
  }
  // pointer operand (R7 / SURVEY O5 step 6)
  uint32_t pk = PK_IMM, ptr = kRegNone;
  if (dpos >= 0 && !(cls & (C_CONSTLOAD | C_SREG | C_MEMLOAD))) {
    const Operand* L[16];
    int nl = 0;
    for (int q = dpos + 1; q < no; q++) if (ops[q].k != T_PRED) L[nl++] = &ops[q];
    const Operand* pick = nullptr;
    auto live_reg = [](const Operand* o) { return o->k == T_REG && reg_live((uint32_t)o->reg); };
    if ((mn.eq("IMAD") || mn.eq("UIMAD")) && has("WIDE")) {
      pick = nl > 2 ? L[2] : nullptr;
    } else if (mn.eq("LEA") || mn.eq("ULEA")) {
      pick = nl > 1 ? L[1] : nullptr;
    } else if (mn.eq("IADD3") || mn.eq("UIADD3")) {
      for (int q = 0; q < nl && !pick; q++) if (L[q]->k == T_CREF) pick = L[q];
      for (int q = 0; q < nl && !pick; q++) if (live_reg(L[q]) && L[q]->reg >= 256) pick = L[q];
      for (int q = 0; q < nl && !pick; q++) if (live_reg(L[q]) && L[q]->reg < 256) pick = L[q];
    } else {
      for (int q = 0; q < nl && !pick; q++) if (live_reg(L[q]) || L[q]->k == T_CREF) pick = L[q];
    }
    if (pick && pick->k == T_CREF) { pk = PK_CONST; cbank = (uint32_t)pick->bank; imm = (int32_t)pick->imm; }
    else if (pick && live_reg(pick)) { pk = PK_REG; ptr = (uint32_t)pick->reg; }
  }
  // backward branch (R13, R28)
  if (op == OP_BRA && no > 0) {
    long long t;
    if (to_int(raw_last, &t)) {
      long long pc = 16LL * (long long)index;
      if (t < pc) {
        long long tidx = t <= 0 ? 0 : (t + 15) / 16;
        flags |= F_BRA_OK;
        imm = (int32_t)tidx;
      }
    }
  }
  // register-pressure inputs (R36, R38)
  lo->exit = mn.eq("EXIT") || mn.eq("RET");
  if (op == OP_BRA) {  // a predicate or register condition before the target may fall through (R38i)
    for (int q = 0; q + 1 < no; q++) lo->brpred |= (ops[q].k == T_PRED && ops[q].predvar) || ops[q].k == T_REG;
    long long t;
    Sv lt = trim(raw_last);
    if (no > 0 && to_int(lt, &t)) lo->target = t;
    else if (lt.n > 4 && lt[0] == '`' && lt[1] == '(' && lt[lt.n - 1] == ')') lo->label.assign(lt.p + 2, lt.n - 3);
  }
  {
    const size_t use0 = lo->uses->size();
    uint32_t srcw = (op == OP_DADD || op == OP_DMUL || op == OP_DFMA || op == OP_DMNMX || mn.eq("DSETP")) ? 2 : 1;
    if (conv) srcw = csw;  // R38e
    const bool store_like = op == OP_STG || op == OP_STS || op == OP_STL || op == OP_ST || op == OP_RED ||
                            op == OP_REDG || op == OP_ATOMG || op == OP_ATOM || op == OP_ATOMS || mn.eq("STSM") ||
                            mn.eq("STTM") || mn.eq("STAS");
    uint32_t dataw = 1;  // data operand width of a store (R36, R38a/d)
    for (int q = 0; q < nm; q++) if (mods[q].eq("64") || is64type(mods[q])) dataw = 2;
    if (mn.eq("STSM")) dataw = has("4") ? 4 : (has("2") ? 2 : 1);
    if (mn.eq("STTM")) dataw = tmem_width(mods, nm);
    for (int q = 0; q < nm; q++) if (mods[q].eq("128") || mods[q].eq("256")) dataw = 4;
    const bool ext = has("E"), wide_imad = op == OP_IMAD && has("WIDE");
    const bool hi_add = op == OP_IMAD && has("HI");  // R38h: 64-bit addend
    const bool target_pair = op == OP_BRX || op == OP_RET || op == OP_CALL || mn.eq("BRXU") || mn.eq("JMX") ||
                             mn.eq("JMXU");  // R38g: 64-bit target address
    int last_mem = -1;  // R38j: .E names the last memory operand
    for (int q = 0; q < no; q++) if (ops[q].k == T_MEM) last_mem = q;
    int srcidx = 0;
    for (int q = 0; q < no; q++) {
      if (q == dpos || q == dpos2) continue;
      const Operand& o = ops[q];
      for (int t = 0; t < o.nregs; t++) {
        const int r = o.regs[t];
        if (r < 0 || r >= 255) continue;  // RZ and uniform registers
        uint32_t w;
        if (o.k == T_MEM) w = (r == o.base && (o.wide || (ext && q == last_mem))) ? 2 : 1;
        else if (o.k == T_CREF) w = 1;
        else if (target_pair) w = 2;
        else if (store_like && q > 0) w = dataw;
        else if (op == OP_HMMA) w = srcidx == 0 ? mma_a : (srcidx == 1 ? mma_b : mma_acc);
        else if ((wide_imad || hi_add) && srcidx == 2) w = 2;
        else w = srcw;
        for (uint32_t k2 = 0; k2 < w && r + (int)k2 < 255; k2++) lo->uses->push_back((uint8_t)(r + k2));
      }
      if (q > last_dst && o.k != T_PRED) srcidx++;
    }
    if (op == OP_CALL) {  // R38g: a call reads R0 and the stack pointer R1
      lo->uses->push_back(0);
      lo->uses->push_back(1);
    }
    // highest GPR touched (the kernel's register count when the dump has no REG:N, R38k)
    for (size_t q = use0; q < lo->uses->size(); q++) lo->maxreg = std::max(lo->maxreg, (int)(*lo->uses)[q]);
    for (uint32_t d : {dst, dst2})
      if (d < 255) lo->maxreg = std::max(lo->maxreg, (int)std::min<uint32_t>(d + dstw - 1, 254));
  }
  if (lo->guarded) flags |= F_PRED;
  if (lo->exit) flags |= F_EXIT;
  if (lo->brpred) flags |= F_BRPRED;
  if (cbank > 31) { *msg = "constant bank > 31"; return false; }
  *out = make_rec(op, flags, aw, dstw, pk, cbank, dst, ptr, s[0], s[1], s[2], s[3], imm);
  (void)lineno;
  return true;
}

int param_base_for(int sm) { return sm >= 100 ? 0x380 : (sm >= 90 ? 0x210 : 0x160); }

struct Segment {
  size_t begin, end;  // byte range (lines after the header)
  long first_line;    // 1-based line number of the first line in range
  int sm;
  std::string name;
  bool header;        // false for an anonymous leading kernel
  int regcount;       // REG:N of a cuobjdump -res-usage block for this function, -1 if none (R38k)
};

// nvdisasm function label ".text.<name>:"
inline bool is_fn_label(Sv t) { return t.n > 7 && starts(t, ".text.") && t[t.n - 1] == ':'; }
// nvdisasm branch label ".L_x_N:"
inline bool is_br_label(Sv t) { return t.n > 3 && starts(t, ".L") && t[t.n - 1] == ':'; }

bool parse_segment(const char* text, const Segment& seg, ParsedKernel* pk, std::string* err) {
  pk->name = seg.name;
  pk->param_base = (uint32_t)param_base_for(seg.sm);
  long lineno = seg.first_line;
  int32_t src_line = -1;
  std::string src_file;
  std::map<std::pair<std::string, int32_t>, int32_t> lkey;  // (file, line) -> kernel-local key
  std::map<std::string, long long> labels;                  // branch label -> pc
  std::vector<std::string> pending;
  std::vector<std::pair<size_t, std::string>> fwd;          // branches to labels not seen yet
  std::vector<std::vector<std::string>> brx_labels;         // BRANCH_TARGETS of each BRX (R38i)
  std::vector<size_t> brx_at;
  int maxreg = -1;
  pk->use_off.assign(1, 0);
  size_t p = seg.begin;
  while (p < seg.end) {
    const char* nl = (const char*)memchr(text + p, '\n', seg.end - p);
    size_t e = nl ? (size_t)(nl - text) : seg.end;
    Sv t = trim(Sv{text + p, e - p});
    long cur = lineno;
    p = e + 1;
    lineno++;
    if (!t.n) continue;
    if (starts(t, "//##")) {  // nvdisasm -g: //## File "f", line N
      size_t at;
      if (contains(t, "line ", &at)) src_line = atoi(std::string(t.p + at + 5, t.n - at - 5).c_str());
      const char* q0 = (const char*)memchr(t.p, '"', t.n);
      const char* q1 = q0 ? (const char*)memchr(q0 + 1, '"', t.n - (size_t)(q0 + 1 - t.p)) : nullptr;
      src_file = q1 ? std::string(q0 + 1, (size_t)(q1 - q0 - 1)) : std::string();
      continue;
    }
    if (is_br_label(t)) {
      pending.emplace_back(t.p, t.n - 1);
      continue;
    }
    if (t.n < 4 || t[0] != '/' || t[1] != '*') continue;
    size_t c = 2;
    while (c + 1 < t.n && !(t[c] == '*' && t[c + 1] == '/')) c++;
    if (c + 1 >= t.n) continue;
    Sv pcs{t.p + 2, c - 2};
    bool hex = pcs.n > 0;
    for (size_t q = 0; q < pcs.n; q++) if (hexv(pcs[q]) < 0) hex = false;
    if (!hex || starts(pcs, "0x")) continue;
    Sv body{t.p + c + 2, t.n - c - 2};
    size_t semi = 0;
    while (semi < body.n && body[semi] != ';') semi++;
    if (semi == body.n) continue;
    long long pc = 0;
    for (size_t q = 0; q < pcs.n; q++) pc = pc * 16 + hexv(pcs[q]);
    if (pc != 16LL * (long long)pk->recs.size()) {
      *err = "line " + std::to_string(cur) + ": pc not 16-strided";
      return false;
    }
    for (auto& lb : pending) labels[lb] = pc;
    pending.clear();
    Sv ins{body.p, semi};
    // nvdisasm annotates an indirect branch with its targets: (*"BRANCH_TARGETS .L_a,.L_b"*) (R38i)
    std::vector<std::string> targets;
    for (size_t q = 0; q + 2 < ins.n; q++)
      if (ins[q] == '(' && ins[q + 1] == '*' && ins[q + 2] == '"') {
        Sv a{ins.p + q, ins.n - q};
        size_t bt;
        if (contains(a, "BRANCH_TARGETS ", &bt)) {
          size_t e = bt + 15;
          while (e < a.n && a[e] != '"') e++;
          Sv list{a.p + bt + 15, e - bt - 15};
          size_t s0 = 0;
          for (size_t k = 0; k <= list.n; k++)
            if (k == list.n || list[k] == ',') {
              Sv lb = trim(Sv{list.p + s0, k - s0});
              if (lb.n) targets.emplace_back(lb.p, lb.n);
              s0 = k + 1;
            }
        }
        ins = trim(Sv{ins.p, q});
        break;
      }
    std::string subst;  // `(.L_x_N) -> 0x<pc> when the label is already known (a backward target)
    const char* bq = (const char*)memchr(ins.p, '`', ins.n);
    if (bq && bq + 1 < ins.p + ins.n && bq[1] == '(') {
      const char* rp = (const char*)memchr(bq, ')', (size_t)(ins.p + ins.n - bq));
      if (rp) {
        auto it = labels.find(std::string(bq + 2, (size_t)(rp - bq - 2)));
        if (it != labels.end()) {
          char hx[32];
          snprintf(hx, sizeof hx, "0x%llx", it->second);
          subst.assign(ins.p, (size_t)(bq - ins.p));
          subst += hx;
          subst.append(rp + 1, (size_t)(ins.p + ins.n - rp - 1));
          ins = Sv{subst.data(), subst.size()};
        }
      }
    }
    Rec r;
    std::string msg;
    LiveOut lo;
    lo.uses = &pk->use_reg;
    if (!pack_line(ins, cur, pk->recs.size(), &r, &msg, &lo)) {
      *err = "line " + std::to_string(cur) + ": " + msg;
      return false;
    }
    pk->use_off.push_back((uint32_t)pk->use_reg.size());
    pk->tgt.push_back(lo.target >= 0 && lo.target % 16 == 0 ? (int32_t)(lo.target / 16) : -1);
    if (lo.target < 0 && !lo.label.empty()) fwd.emplace_back(pk->recs.size(), lo.label);
    if (r_op(r) == OP_BRX && !targets.empty()) {  // multi-target entry, resolved at the end
      pk->tgt.back() = -2 - (int32_t)brx_at.size();
      brx_at.push_back(pk->recs.size());
      brx_labels.push_back(std::move(targets));
    }
    maxreg = std::max(maxreg, lo.maxreg);
    pk->recs.push_back(r);
    pk->lines.push_back(src_line);
    int32_t key = -1;
    if (src_line >= 0) {
      auto ins_it = lkey.emplace(std::make_pair(src_file, src_line), (int32_t)lkey.size());
      key = ins_it.first->second;
    }
    pk->lkeys.push_back(key);
  }
  pk->n_lkeys = (uint32_t)lkey.size();
  for (auto& pl : pending) labels[pl] = 16LL * (long long)pk->recs.size();  // labels after the last instruction
  for (auto& f : fwd) {  // forward label targets (backward ones were substituted in place)
    auto it = labels.find(f.second);
    if (it != labels.end()) pk->tgt[f.first] = (int32_t)(it->second / 16);
  }
  // indirect-branch successor lists (R38i): kernel-local instruction indices, CSR
  pk->xtgt_off.assign(1, 0);
  for (size_t b = 0; b < brx_at.size(); b++) {
    for (auto& lb : brx_labels[b]) {
      auto it = labels.find(lb);
      if (it != labels.end() && it->second / 16 < (long long)pk->recs.size()) pk->xtgt.push_back((int32_t)(it->second / 16));
    }
    pk->xtgt_off.push_back((uint32_t)pk->xtgt.size());
  }
  // the kernel's register count (R38k): the dump's REG:N, else one past the highest GPR touched
  pk->nregs = seg.regcount > 0 ? (uint32_t)seg.regcount : (uint32_t)(maxreg + 1);
  return true;
}

bool is_instr_line(Sv t) {
  if (t.n < 4 || t[0] != '/' || t[1] != '*') return false;
  size_t c = 2;
  while (c + 1 < t.n && !(t[c] == '*' && t[c + 1] == '/')) c++;
  if (c + 1 >= t.n || c == 2) return false;
  for (size_t q = 2; q < c; q++) if (hexv(t[q]) < 0) return false;
  if (t[2] == '0' && t[3] == 'x') return false;
  Sv body{t.p + c + 2, t.n - c - 2};
  for (size_t q = 0; q < body.n; q++) if (body[q] == ';') return true;
  return false;
}

// Pass 1 in parallel: only lines containing one of these can change the segment state (the
// header state machine below), plus the first instruction line of a module without headers.
struct Cand {
  size_t b, e;  // line [b, e)
  long lineno;  // 1-based
};
void find_candidates(const char* text, size_t b0, size_t e0, std::vector<Cand>* out, long* nlines) {
  static const char* const pats[] = {"Function", "REG:", "code for sm_", ".target", ".text."};
  std::vector<size_t> hits;
  for (const char* pt : pats) {
    const size_t m = strlen(pt);
    size_t q = b0;
    while (q < e0) {
      const void* f = memmem(text + q, e0 - q, pt, m);
      if (!f) break;
      const size_t at = (size_t)((const char*)f - text);
      hits.push_back(at);
      q = at + 1;
    }
  }
  // the first instruction line of the range (a module whose instructions precede any header)
  for (size_t q = b0; q < e0;) {
    const char* nl = (const char*)memchr(text + q, '\n', e0 - q);
    const size_t e = nl ? (size_t)(nl - text) : e0;
    Sv t = trim(Sv{text + q, e - q});
    if (t.n && !starts(t, "//##") && is_instr_line(t)) { hits.push_back(q); break; }
    q = e + 1;
  }
  std::sort(hits.begin(), hits.end());
  // lines of the hits (deduplicated), with line numbers relative to b0
  long line = 0;
  size_t pos = b0, lb = b0;  // lb: start of the line holding pos
  size_t last_b = ~(size_t)0;
  for (size_t h : hits) {
    while (pos < h) {  // advance to the line of h, counting newlines
      const char* nl = (const char*)memchr(text + pos, '\n', h - pos);
      if (!nl) { pos = h; break; }
      line++;
      pos = (size_t)(nl - text) + 1;
      lb = pos;
    }
    if (lb == last_b) continue;
    const char* nl = (const char*)memchr(text + lb, '\n', e0 - lb);
    out->push_back(Cand{lb, nl ? (size_t)(nl - text) : e0, line});
    last_b = lb;
  }
  // total lines of the range: newlines after pos
  for (size_t q = pos; q < e0;) {
    const char* nl = (const char*)memchr(text + q, '\n', e0 - q);
    if (!nl) break;
    line++;
    q = (size_t)(nl - text) + 1;
  }
  *nlines = line;
}

}  // namespace

bool parse_sass(const char* text, size_t len, int n_threads, std::vector<ParsedKernel>* out, std::string* err) {
  // pass 1: segments. The ranges (cut after a newline) are scanned in parallel for candidate
  // lines; the header state machine then runs over the candidates in text order, exactly as it
  // would over every line (the other lines take none of its branches).
  // ranges of at least 1 MB (GS_PARSE_RANGE_BYTES overrides it: tests cut tiny inputs finely)
  static const size_t min_range = [] {
    const char* v = getenv("GS_PARSE_RANGE_BYTES");
    return v && atoll(v) > 0 ? (size_t)atoll(v) : (size_t)1 << 20;
  }();
  const int nr = (int)std::max<size_t>(1, std::min<size_t>((size_t)n_threads, len / min_range + 1));
  std::vector<size_t> cut(nr + 1, len);
  cut[0] = 0;
  for (int r = 1; r < nr; r++) {
    size_t q = std::max(cut[r - 1], len * (size_t)r / (size_t)nr);
    const char* nl = q < len ? (const char*)memchr(text + q, '\n', len - q) : nullptr;
    cut[r] = nl ? (size_t)(nl - text) + 1 : len;
  }
  std::vector<std::vector<Cand>> cands(nr);
  std::vector<long> nlines(nr, 0);
  {
    std::vector<std::thread> th;
    for (int r = 1; r < nr; r++)
      th.emplace_back([&, r]() { find_candidates(text, cut[r], cut[r + 1], &cands[r], &nlines[r]); });
    find_candidates(text, cut[0], cut[1], &cands[0], &nlines[0]);
    for (auto& t : th) t.join();
  }
  std::vector<Segment> segs;
  std::map<std::string, int> res_regs;  // cuobjdump -res-usage: " Function <name>:" / "  REG:N ..." (R38k)
  std::string res_fn;
  int sm = 100;
  long line0 = 1;  // line number of the first line of range r
  for (int r = 0; r < nr; r++) {
    for (const Cand& cd : cands[r]) {
      const size_t p = cd.b, e = cd.e;
      const long lineno = line0 + cd.lineno;
      Sv t = trim(Sv{text + p, e - p});
      size_t at;
      if (!t.n) continue;
      if (starts(t, "Function ") && t[t.n - 1] == ':' && !contains(t, "Function :")) {
        res_fn.assign(t.p + 9, t.n - 10);
      } else if (!res_fn.empty() && starts(t, "REG:")) {
        res_regs[res_fn] = atoi(std::string(t.p + 4, std::min<size_t>(t.n - 4, 12)).c_str());
        res_fn.clear();
      } else if (contains(t, "code for sm_", &at)) {
        sm = atoi(std::string(t.p + at + 12, t.n - at - 12).c_str());
      } else if (contains(t, ".target") && contains(t, "sm_", &at)) {
        sm = atoi(std::string(t.p + at + 3, t.n - at - 3).c_str());
      } else if (contains(t, "Function :", &at) || is_fn_label(t)) {
        if (!segs.empty()) segs.back().end = p;
        Segment sg;
        sg.begin = e + 1 > len ? len : e + 1;
        sg.end = len;
        sg.first_line = lineno + 1;
        sg.sm = sm;
        Sv nm = is_fn_label(t) ? Sv{t.p + 6, t.n - 7} : trim(Sv{t.p + at + 10, t.n - at - 10});
        sg.name.assign(nm.p, nm.n);
        sg.header = true;
        auto rr = res_regs.find(sg.name);
        sg.regcount = rr == res_regs.end() ? -1 : rr->second;
        segs.push_back(sg);
      } else if (segs.empty() && !starts(t, "//##") && is_instr_line(t)) {
        Segment sg;  // instructions before any Function header: one anonymous kernel
        sg.begin = 0;
        sg.end = len;
        sg.first_line = 1;
        sg.sm = sm;
        sg.name = "<anonymous>";
        sg.header = false;
        sg.regcount = -1;
        segs.push_back(sg);
      }
    }
    line0 += nlines[r];
  }
  // a later "code for"/".target" line inside a segment applies to the next Function only; the
  // per-segment sm was captured when its header was seen.
  out->assign(segs.size(), ParsedKernel());
  std::vector<std::string> errs(segs.size());
  std::atomic<size_t> next(0);
  std::atomic<bool> failed(false);
  auto worker = [&]() {
    for (;;) {
      size_t k = next.fetch_add(1);
      if (k >= segs.size() || failed.load()) return;
      if (!parse_segment(text, segs[k], &(*out)[k], &errs[k])) failed = true;
    }
  };
  int nt = std::max(1, std::min<int>(n_threads, (int)segs.size()));
  std::vector<std::thread> th;
  for (int i = 1; i < nt; i++) th.emplace_back(worker);
  worker();
  for (auto& t : th) t.join();
  for (size_t k = 0; k < segs.size(); k++)
    if (!errs[k].empty()) { *err = errs[k]; return false; }
  return true;
}

}  // namespace gs
