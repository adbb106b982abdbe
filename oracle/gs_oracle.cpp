// gs_oracle.cpp — the CPU ORACLE for batched bottleneck attribution (GPUscout, SC-W 2023).
//
// *** TEST INFRASTRUCTURE ONLY. ***  Only tests/, __graft_entry__.smoke() and bench.py's
// cpu_baseline / --impl reference legs may build, call or execute this program. It shares no
// code, header, table or helper with the CUDA path (paper_conf_sc_senvs23_b200/csrc); the two
// are written independently from the same reading of the paper.
//
// Plain, slow, obviously-correct: single-threaded, std::vector / std::map / std::sort, linear
// scans, its own SASS text parser. Every step cites the PAPER.md passage (P:line, section) it
// follows; where the paper is silent the DESIGN.md reading number is given (e.g. [R5]).
//
// Steps (SURVEY §8c O1–O15):
//   O1  parse cuobjdump/nvdisasm SASS text                      P:209-213 §2.1
//   O2  per-instruction register effects (dst, width, sources)   P:211-213 ("destination (+source) register numbers")
//   O3  reaching definition = last earlier writer (linear order)  P:446-448 §3.2 ("previous SASS instruction executed by the register")
//   O4  loop depth from backward branches                        P:640-645 §4.3, §4.4
//   O5  bounded backward def-use trace of an address register    P:446-448, §4.2; north_star
//   O6  VEC   vectorisable 32-bit global loads                   P:510-532 §4.1, Listing 1
//   O7  SPILL local-memory spills STL/LDL + cause                  P:565-583 §4.2
//   O8  SHMEM shared-memory candidates                           P:626-645 §4.3
//   O9  GATOM global atomics                                     P:669-696 §4.4
//   O10 RO    read-only / __restrict__ candidates                P:698-715 §4.5
//   O11 TEX   texture candidates                                 P:717-744 §4.6
//   O12 CONV  datatype conversions                               P:746-761 §4.7
//   O13 per-PC x stall-reason histogram of PC samples            P:215-227 §2.2
//       (raw samples, pre-aggregated count records [R35], CUPTI PC-sampling records [R39])
//   O14 join of the histogram onto flagged sites
//       join=pc (default), line ([R33]), consumer ([R37], SURVEY [probe 9])
//   O15 ranking (total order on integers)                        [R20]
//   O16 register pressure: live GPRs per instruction (--liveness) P:541-554, P:452 [R36, R38]
//
// Output: the canonical result text on stdout or --out.
#include <algorithm>
#include <chrono>
#include <cstdint>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <map>
#include <set>
#include <string>
#include <vector>

namespace {

// ---------------------------------------------------------------- registers
// One id space: GPR R0..R254 -> 0..254, RZ -> 255; UR0..UR62 -> 256..318, URZ -> 319.
const int kRZ = 255, kURZ = 319, kNoReg = -1;
bool is_zero_reg(int r) { return r == kRZ || r == kURZ; }
bool is_ur(int r) { return r >= 256; }
std::string reg_name(int r) {
  char b[16];
  if (r < 256) snprintf(b, sizeof b, r == kRZ ? "RZ" : "R%d", r);
  else snprintf(b, sizeof b, r == kURZ ? "URZ" : "UR%d", r - 256);
  return b;
}

// ---------------------------------------------------------------- operands
enum OpndKind { K_REG, K_PRED, K_CREF, K_MEM, K_IMM, K_OTHER };
struct Opnd {
  OpndKind kind = K_OTHER;
  int reg = kNoReg;            // K_REG: register id
  std::vector<int> regs;       // every register token inside the operand (any kind)
  int cbank = 0;               // K_CREF: bank
  long long coff = 0;          // K_CREF: offset (immediate part)
  int base = kNoReg;           // K_MEM: first register term of the address
  long long off = 0;           // K_MEM: sum of immediate terms
  bool wide = false;           // K_MEM: the base is a 64-bit pair (Rb.64)
  bool pred_var = false;       // K_PRED: a real predicate (not PT / UPT)
};

std::string trim(const std::string& s) {
  size_t a = s.find_first_not_of(" \t\r\n"), b = s.find_last_not_of(" \t\r\n");
  return a == std::string::npos ? std::string() : s.substr(a, b - a + 1);
}

// Parse a bare register token (prefixes - ! ~ | already stripped), e.g. "R4.64", "UR6", "RZ".
bool parse_reg(const std::string& t0, int* out) {
  std::string t = t0;
  size_t dot = t.find('.');
  if (dot != std::string::npos) t = t.substr(0, dot);
  while (!t.empty() && t.back() == '|') t.pop_back();
  bool ur = false;
  size_t p = 0;
  if (t.size() >= 2 && t[0] == 'U' && t[1] == 'R') { ur = true; p = 2; }
  else if (!t.empty() && t[0] == 'R') p = 1;
  else return false;
  std::string rest = t.substr(p);
  if (rest == "Z") { *out = ur ? kURZ : kRZ; return true; }
  if (rest.empty() || rest.size() > 3) return false;
  for (char c : rest) if (c < '0' || c > '9') return false;
  int n = atoi(rest.c_str());
  if (ur ? n > 62 : n > 254) return false;
  *out = ur ? 256 + n : n;
  return true;
}

std::string strip_prefix(const std::string& t) {
  size_t i = 0;
  while (i < t.size() && (t[i] == '-' || t[i] == '!' || t[i] == '~' || t[i] == '|')) i++;
  return t.substr(i);
}

bool parse_int(const std::string& t0, long long* v) {
  std::string t = trim(t0);
  bool neg = false;
  if (!t.empty() && (t[0] == '-' || t[0] == '+')) { neg = t[0] == '-'; t = t.substr(1); }
  if (t.empty()) return false;
  char* end = nullptr;
  long long x;
  if (t.size() > 2 && t[0] == '0' && (t[1] == 'x' || t[1] == 'X')) x = strtoll(t.c_str() + 2, &end, 16);
  else x = strtoll(t.c_str(), &end, 10);
  if (*end) return false;
  *v = neg ? -x : x;
  return true;
}

// Sum immediates and collect registers of a bracket body like "R4.64+-0x10" or "R11+UR4".
void parse_bracket(const std::string& body, Opnd* o, bool first_reg_is_base) {
  size_t s = 0;
  std::string b = body;
  while (s <= b.size()) {
    size_t e = b.find('+', s);
    if (e == std::string::npos) e = b.size();
    std::string term = trim(b.substr(s, e - s));
    if (!term.empty()) {
      int r;
      long long v;
      if (parse_reg(strip_prefix(term), &r)) {
        o->regs.push_back(r);
        if (first_reg_is_base && o->base == kNoReg) o->base = r;
      } else if (parse_int(term, &v)) {
        o->off += v;
      }
    }
    s = e + 1;
  }
}

Opnd parse_operand(const std::string& raw) {
  Opnd o;
  std::string t = trim(raw);
  std::string u = strip_prefix(t);
  // constant-bank reference c[bank][off]   (may carry a register inside the second bracket)
  if (u.size() > 2 && u[0] == 'c' && u[1] == '[') {
    o.kind = K_CREF;
    size_t a = u.find(']');
    long long bank = 0;
    parse_int(u.substr(2, a - 2), &bank);
    o.cbank = (int)bank;
    size_t b0 = u.find('[', a), b1 = u.find(']', b0 == std::string::npos ? a : b0);
    if (b0 != std::string::npos && b1 != std::string::npos) {
      Opnd tmp;
      parse_bracket(u.substr(b0 + 1, b1 - b0 - 1), &tmp, false);
      o.coff = tmp.off;
      o.regs = tmp.regs;
    }
    return o;
  }
  // memory operand [..], desc[URx][..], [R11+UR4]
  if (u.find('[') != std::string::npos) {
    o.kind = K_MEM;
    size_t last_open = u.rfind('[');
    size_t last_close = u.find(']', last_open);
    // registers of any earlier bracket (desc[URd]) are sources, not the base
    size_t p = 0;
    while (true) {
      size_t a = u.find('[', p);
      if (a == std::string::npos || a == last_open) break;
      size_t c = u.find(']', a);
      Opnd tmp;
      parse_bracket(u.substr(a + 1, c - a - 1), &tmp, false);
      for (int r : tmp.regs) o.regs.push_back(r);
      p = c + 1;
    }
    Opnd inner;
    const std::string ib = u.substr(last_open + 1, last_close - last_open - 1);
    parse_bracket(ib, &inner, true);
    o.wide = ib.find(".64") != std::string::npos;
    o.base = inner.base;
    o.off = inner.off;
    for (int r : inner.regs) o.regs.push_back(r);
    return o;
  }
  int r;
  if (parse_reg(u, &r)) { o.kind = K_REG; o.reg = r; o.regs.push_back(r); return o; }
  {  // predicates P0..P6, PT, UP0..UP6, UPT (optionally negated)
    std::string p = u;
    if (p.size() >= 2 && p[0] == 'U' && p[1] == 'P') p = p.substr(2);
    else if (!p.empty() && p[0] == 'P') p = p.substr(1);
    else p = "#";
    if (p == "T" || (p.size() == 1 && p[0] >= '0' && p[0] <= '7')) {
      o.kind = K_PRED;
      o.pred_var = p != "T";
      return o;
    }
  }
  long long v;
  if (parse_int(t, &v)) { o.kind = K_IMM; return o; }
  o.kind = K_OTHER;  // SR_TID.X, floats, B0, 2D, PR ...  (never registers)
  return o;
}

// ---------------------------------------------------------------- instructions
struct Instr {
  int pc = 0;
  int line = -1;                  // source line from //## File ..., line N
  std::string file;               // ... and its file (a source line is the pair (file, line), R33)
  std::string bra_label;          // nvdisasm: BRA `(.L_x_N) target label, resolved per kernel
  std::vector<std::string> brx_labels;  // nvdisasm: BRX ... (*"BRANCH_TARGETS .L_a,.L_b"*) (R38i)
  std::vector<long long> brx_targets;   // ... resolved to pcs
  bool guarded = false;           // @Pn / @!Pn guard (not @PT)
  std::string op;                 // base mnemonic
  std::vector<std::string> mods;  // modifiers after the first '.'
  std::vector<Opnd> ops;
  int dst = kNoReg, dst_w = 0, dst_pos = -1;
  int dst2 = kNoReg, dst2_pos = -1;  // second destination quad of a .256 load (R38a)
  std::vector<int> srcs;          // register sources (no RZ/URZ), O2
  int mem = -1;                   // index of the memory operand in ops
  long long bra_target = -1;      // BRA immediate target pc
  bool has_mod(const char* m) const {
    for (auto& s : mods) if (s == m) return true;
    return false;
  }
};

struct Kernel {
  std::string name;
  int param_base = 0x380;
  int regcount = -1;                  // REG:N of a cuobjdump -res-usage block, if the dump has one (R38k)
  std::vector<Instr> ins;
  size_t first_slot = 0;
  std::map<std::string, int> labels;  // nvdisasm ".L_x_N:" -> pc of the next instruction
};

bool op_in(const std::string& op, std::initializer_list<const char*> l) {
  for (auto* s : l) if (op == s) return true;
  return false;
}

// ---- register widths (R24, revised for sm_100a by R38; pinned to nvdisasm -lrm narrow) ----
bool is_64type(const std::string& m) { return m == "F64" || m == "S64" || m == "U64"; }
bool is_int_type(const std::string& m) {
  return m == "S64" || m == "U64" || m == "S32" || m == "U32" || m == "S16" || m == "U16" || m == "S8" || m == "U8";
}
bool is_float_type(const std::string& m) {
  return m == "F64" || m == "F32" || m == "F16" || m == "BF16" || m == "TF32" || m == "E4M3" || m == "E5M2";
}
bool is_type(const std::string& m) { return is_int_type(m) || is_float_type(m); }

// R38e conversions: which type modifier names the destination and which the source.
//   F2F, I2I: first type = destination, second = source (F2F.F32.F64);
//   I2F, I2FP: the float type is the destination, the integer type the source (I2F.U64.RP: u64 -> f32);
//   F2I, F2IP: the integer type is the destination, the float type the source (F2I.F64.TRUNC: f64 -> s32).
// Returns the register widths {dst, src} (2 for a 64-bit type, else 1).
std::pair<int, int> conv_widths(const Instr& I) {
  std::vector<std::string> t;
  for (auto& m : I.mods) if (is_type(m)) t.push_back(m);
  std::string d, s;
  if (op_in(I.op, {"F2F", "I2I"})) {
    if (t.size() >= 1) d = t[0];
    if (t.size() >= 2) s = t[1];
  } else if (op_in(I.op, {"I2F", "I2FP"})) {
    for (auto& m : t) (is_float_type(m) ? d : s) = m;
  } else if (op_in(I.op, {"F2I", "F2IP"})) {
    for (auto& m : t) (is_int_type(m) ? d : s) = m;
  } else if (I.op == "F2FP") {
    if (t.size() >= 1) d = t[0];
    if (t.size() >= 2) s = t[1];
  }
  return {is_64type(d) ? 2 : 1, is_64type(s) ? 2 : 1};
}

// R38c warp-level MMA fragments: HMMA.<m><n><k>.<acc>[.<in>] on an m16n8kK tile holds, per thread,
// A = 16*K*b/1024 and B = 8*K*b/1024 registers (b = input element bits: F16/BF16 16 (default), TF32
// 32, E4M3/E5M2 8) and C = D = 4 registers for an F32 accumulator, 2 for F16.
struct MmaRegs { int a = 1, b = 1, acc = 1; };
MmaRegs mma_regs(const Instr& I) {
  MmaRegs r;
  int K = 8, bits = 16;
  std::string acc;
  for (size_t q = 0; q < I.mods.size(); q++) {
    const std::string& m = I.mods[q];
    if (q == 0 && m.size() >= 4 && isdigit((unsigned char)m[0])) K = atoi(m.c_str() + 3);  // "16816" -> 16, "1688" -> 8
    else if (acc.empty() && is_float_type(m)) acc = m;
    else if (m == "TF32") bits = 32;
    else if (m == "E4M3" || m == "E5M2") bits = 8;
  }
  r.a = std::max(1, 16 * K * bits / 1024);
  r.b = std::max(1, 8 * K * bits / 1024);
  r.acc = acc == "F16" ? 2 : 4;
  return r;
}

// R38d tensor-memory loads/stores (tcgen05.ld/st): LDTM[.<shape>].x<N>; registers per thread per
// repetition: 32dp32bit (no shape modifier) 1, 16dp32bit 1, 16dp64bit 1, 16dp128bit 2, 16dp256bit 4.
int tmem_regs(const Instr& I) {
  int per = 1, x = 1;
  for (auto& m : I.mods) {
    if (m == "16dp128bit") per = 2;
    else if (m == "16dp256bit") per = 4;
    else if (m.size() > 1 && m[0] == 'x' && isdigit((unsigned char)m[1])) x = atoi(m.c_str() + 1);
  }
  return per * x;
}

// O2 destination width table (DESIGN.md §3 table W: R24 as revised by R38).
int dst_width(const Instr& I) {
  for (auto& m : I.mods) if (m == "256") return 4;      // R38a: each of the two destination quads
  for (auto& m : I.mods) if (m == "128") return 4;
  if (I.op == "HMMA") return mma_regs(I).acc;             // R38c
  if (I.op == "LDSM") {
    if (I.has_mod("4")) return 4;
    if (I.has_mod("2")) return 2;
    return 1;
  }
  if (I.op == "LDTM") return tmem_regs(I);                // R38d
  for (auto& m : I.mods) if (m == "64" || m == "WIDE") return 2;
  if (I.op == "CS2R") return I.has_mod("32") ? 1 : 2;     // R38b: CS2R writes a pair unless .32
  if (I.op == "LEPC") return 2;                           // R38b: a 64-bit program counter
  if (op_in(I.op, {"DADD", "DMUL", "DFMA", "DMNMX"})) return 2;
  if (op_in(I.op, {"F2F", "I2F", "F2I", "I2I", "I2FP", "F2IP", "F2FP"})) return conv_widths(I).first;  // R38e
  return 1;
}

// R38f opcodes whose register operands are all sources (a first register operand is not a
// destination): WARPSYNC Rmask, BRX/JMX Rtarget, RET Rreturn, CALL Rtarget, NANOSLEEP Rns, BAR ... Rn.
bool no_register_dst(const std::string& op) {
  return op_in(op, {"WARPSYNC", "BRX", "BRXU", "JMX", "JMXU", "RET", "CALL", "NANOSLEEP", "BAR", "YIELD", "BPT"});
}

// O2: decode dst and sources.
void decode_effects(Instr& I) {
  int d = -1;
  if (no_register_dst(I.op)) d = -1;
  else if (!I.ops.empty() && I.ops[0].kind == K_REG) d = 0;
  else if (I.ops.size() >= 2 && I.ops[0].kind == K_PRED && I.ops[1].kind == K_REG && I.op != "FCHK")
    d = 1;  // SHFL PT, R0 ... ; ATOMG PT, R2 ... ; LOP3.LUT P0, R5 ...
  int last_dst = d;
  if (d >= 0) {
    I.dst_pos = d;
    I.dst = I.ops[d].reg;
    I.dst_w = dst_width(I);
    // R38a: a 256-bit load (LDG.E.ENL2.256 Ra, Rb, [..]) writes two register quads Ra and Rb
    if (I.has_mod("256") && (size_t)d + 1 < I.ops.size() && I.ops[d + 1].kind == K_REG) {
      I.dst2_pos = d + 1;
      I.dst2 = I.ops[d + 1].reg;
      last_dst = d + 1;
    }
  }
  for (size_t k = (size_t)(last_dst + 1); k < I.ops.size(); k++)
    for (int r : I.ops[k].regs)
      if (!is_zero_reg(r)) I.srcs.push_back(r);
  for (size_t k = 0; k < I.ops.size(); k++)
    if (I.ops[k].kind == K_MEM) { I.mem = (int)k; break; }
}

// ---------------------------------------------------------------- O1 parser
struct ParseError { std::string msg; };

int arch_param_base(int sm) { return sm >= 100 ? 0x380 : (sm >= 90 ? 0x210 : 0x160); }

// Accepts cuobjdump -sass text ("Function : name" headers, hex branch targets) and nvdisasm text
// (".text.name:" labels, "//## File "f", line N" with -g, branch targets as `(.L_x_N) labels).
std::vector<Kernel> parse_sass(const std::string& text) {
  std::vector<Kernel> ks;
  int cur_sm = 100, line_no = 0, src_line = -1;
  std::string src_file;
  std::vector<std::string> pending;  // labels waiting for their instruction
  std::map<std::string, int> res_regs;  // cuobjdump -res-usage: function name -> REG:N (R38k)
  std::string res_fn;
  auto new_kernel = [&](const std::string& name) {
    Kernel k;
    k.name = name;
    k.param_base = arch_param_base(cur_sm);
    auto rr = res_regs.find(name);
    if (rr != res_regs.end()) k.regcount = rr->second;
    ks.push_back(k);
    src_line = -1;
    src_file.clear();
    pending.clear();
  };
  size_t p = 0;
  while (p < text.size()) {
    size_t e = text.find('\n', p);
    if (e == std::string::npos) e = text.size();
    std::string L = text.substr(p, e - p);
    p = e + 1;
    line_no++;
    std::string t = trim(L);
    if (t.empty()) continue;
    size_t cf = t.find("code for sm_");
    if (cf != std::string::npos) { cur_sm = atoi(t.c_str() + cf + 12); continue; }
    size_t tg = t.find(".target");
    if (tg != std::string::npos && t.find("sm_") != std::string::npos) {
      cur_sm = atoi(t.c_str() + t.find("sm_") + 3);
      continue;
    }
    // cuobjdump -res-usage block: " Function <name>:" then "  REG:N STACK:..." (R38k)
    if (t.rfind("Function ", 0) == 0 && t.size() > 10 && t.back() == ':' && t.find("Function :") == std::string::npos) {
      res_fn = t.substr(9, t.size() - 10);
      continue;
    }
    if (!res_fn.empty() && t.rfind("REG:", 0) == 0) {
      res_regs[res_fn] = atoi(t.c_str() + 4);
      res_fn.clear();
      continue;
    }
    size_t fn = t.find("Function :");
    if (fn != std::string::npos) {
      new_kernel(trim(t.substr(fn + 10)));
      continue;
    }
    if (t.size() > 7 && t.rfind(".text.", 0) == 0 && t.back() == ':') {  // nvdisasm function label
      new_kernel(t.substr(6, t.size() - 7));
      continue;
    }
    if (t.size() > 3 && t.rfind(".L", 0) == 0 && t.back() == ':') {  // nvdisasm branch label
      pending.push_back(t.substr(0, t.size() - 1));
      continue;
    }
    if (t.rfind("//##", 0) == 0) {  // nvdisasm -g line info: //## File "f", line N
      size_t ln = t.find("line ");
      if (ln != std::string::npos) src_line = atoi(t.c_str() + ln + 5);
      size_t q0 = t.find('"'), q1 = q0 == std::string::npos ? q0 : t.find('"', q0 + 1);
      src_file = q1 == std::string::npos ? std::string() : t.substr(q0 + 1, q1 - q0 - 1);
      continue;
    }
    if (t.size() < 4 || t[0] != '/' || t[1] != '*') continue;
    size_t c = t.find("*/");
    if (c == std::string::npos) continue;
    std::string pcs = t.substr(2, c - 2);
    bool hex = !pcs.empty();
    for (char ch : pcs) if (!isxdigit((unsigned char)ch)) hex = false;
    if (!hex || pcs.rfind("0x", 0) == 0) continue;  // "/* 0x... */" encoding-only line
    std::string body = t.substr(c + 2);
    size_t semi = body.find(';');
    if (semi == std::string::npos) continue;
    body = trim(body.substr(0, semi));
    // nvdisasm annotates indirect branches with their targets: (*"BRANCH_TARGETS .L_a,.L_b"*) (R38i)
    std::vector<std::string> brx_labels;
    size_t ann = body.find("(*\"");
    if (ann != std::string::npos) {
      std::string a = body.substr(ann);
      body = trim(body.substr(0, ann));
      size_t bt = a.find("BRANCH_TARGETS ");
      if (bt != std::string::npos) {
        std::string list = a.substr(bt + 15);
        list = list.substr(0, list.find('"'));
        size_t s = 0;
        while (s <= list.size()) {
          size_t e = list.find(',', s);
          if (e == std::string::npos) e = list.size();
          std::string lb = trim(list.substr(s, e - s));
          if (!lb.empty()) brx_labels.push_back(lb);
          s = e + 1;
        }
      }
    }
    if (ks.empty()) new_kernel("<anonymous>");  // instructions without a header (e.g. a paper listing)
    Kernel& K = ks.back();
    Instr I;
    I.pc = (int)strtol(pcs.c_str(), nullptr, 16);
    I.line = src_line;
    I.file = src_file;
    if ((size_t)I.pc != K.ins.size() * 16)
      throw ParseError{"line " + std::to_string(line_no) + ": pc not 16-strided"};
    for (auto& lb : pending) K.labels[lb] = I.pc;
    pending.clear();
    // guard predicate
    if (!body.empty() && body[0] == '@') {
      I.guarded = body.rfind("@PT", 0) != 0 && body.rfind("@UPT", 0) != 0;
      size_t sp = body.find_first_of(" \t");
      body = trim(body.substr(sp));
    }
    size_t sp = body.find_first_of(" \t");
    std::string opc = sp == std::string::npos ? body : body.substr(0, sp);
    std::string rest = sp == std::string::npos ? "" : trim(body.substr(sp));
    size_t d0 = opc.find('.');
    I.op = opc.substr(0, d0);
    while (d0 != std::string::npos) {
      size_t d1 = opc.find('.', d0 + 1);
      I.mods.push_back(opc.substr(d0 + 1, d1 == std::string::npos ? std::string::npos : d1 - d0 - 1));
      d0 = d1;
    }
    // split operands at top-level commas; an operand list without a comma between two operands
    // ("RET.REL.NODEC R2 0x0", "BRX R4 -0x43d0") is split at top-level blanks as well (R38i)
    std::vector<std::string> raw;
    int depth = 0;
    std::string cur;
    for (char ch : rest) {
      if (ch == '[' || ch == '{') depth++;
      if (ch == ']' || ch == '}') depth--;
      if (ch == ',' && depth == 0) { raw.push_back(cur); cur.clear(); }
      else if ((ch == ' ' || ch == '\t') && depth == 0 && !trim(cur).empty()) { raw.push_back(cur); cur.clear(); }
      else if ((ch == ' ' || ch == '\t') && depth == 0) continue;
      else cur += ch;
    }
    if (!trim(cur).empty()) raw.push_back(cur);
    for (auto& r : raw) I.ops.push_back(parse_operand(r));
    decode_effects(I);
    if (I.op == "BRA" && !raw.empty()) {
      long long v;
      std::string last = trim(raw.back());
      if (parse_int(last, &v)) I.bra_target = v;
      else if (last.size() > 4 && last.rfind("`(", 0) == 0 && last.back() == ')')
        I.bra_label = last.substr(2, last.size() - 3);
    }
    I.brx_labels = brx_labels;
    K.ins.push_back(I);
  }
  // nvdisasm label targets: a label names the pc of the instruction after it (R28)
  for (auto& k : ks)
    for (auto& I : k.ins) {
      if (!I.bra_label.empty()) {
        auto it = k.labels.find(I.bra_label);
        if (it != k.labels.end()) I.bra_target = it->second;
      }
      for (auto& lb : I.brx_labels) {
        auto it = k.labels.find(lb);
        if (it != k.labels.end()) I.brx_targets.push_back(it->second);
      }
    }
  size_t slot = 0;
  for (auto& k : ks) { k.first_slot = slot; slot += k.ins.size(); }
  return ks;
}

// ---------------------------------------------------------------- opcode classes
bool is_constload(const std::string& op) { return op_in(op, {"LDC", "LDCU", "ULDC"}); }
bool is_sreg(const std::string& op) { return op_in(op, {"S2R", "S2UR", "CS2R"}); }
bool is_memload(const std::string& op) {
  return op_in(op, {"LDG", "LDL", "LDS", "LD", "LDSM", "ATOM", "ATOMG", "ATOMS", "TLD", "TLD4",
                    "TLDS", "TEX", "TMML", "TXD", "TXQ", "SULD", "SUATOM", "LDTM"});
}
bool is_conv(const std::string& op) {
  return op_in(op, {"F2F", "F2I", "I2F", "I2I", "I2FP", "F2IP", "F2FP"});
}
bool is_arith(const Instr& I) {
  if (I.op == "IMAD") return I.mods.empty() || I.mods[0] != "MOV";
  return op_in(I.op, {"FADD", "FMUL", "FFMA", "FMNMX", "DADD", "DMUL", "DFMA", "HADD2", "HMUL2",
                      "HFMA2", "MUFU", "IADD3", "VIADD", "IMUL", "IMNMX", "VIMNMX", "IABS"});
}
bool is_gatom(const std::string& op) { return op_in(op, {"ATOMG", "ATOM", "RED", "REDG"}); }
bool is_store_class(const std::string& op) {
  return op_in(op, {"STG", "ST", "ATOMG", "ATOM", "RED", "REDG", "SUST"});
}
bool is_traced_memop(const std::string& op) {
  return op_in(op, {"LDG", "LDL", "STL", "STG", "ST", "ATOMG", "ATOM", "RED", "REDG", "SUST"});
}
// access width in bits of a memory instruction (reading #2)
int access_bits(const Instr& I) {
  for (auto& m : I.mods) {
    if (m == "U8" || m == "S8") return 8;
    if (m == "U16" || m == "S16") return 16;
    if (m == "64") return 64;
    if (m == "128") return 128;
    if (m == "256") return 256;  // sm_100a LDG.E.ENL2.256: two register quads (R38a)
  }
  return 32;
}

// ---------------------------------------------------------------- O5 traces
enum TermKind { T_NONE, T_PARAM, T_CONST, T_ENTRY, T_SREG, T_MEMORY, T_IMM, T_TRUNC };
struct Trace {
  TermKind kind = T_NONE;
  long long value = 0;  // PARAM: offset; CONST: bank<<32|off; ENTRY: reg; SREG/MEMORY: idx
  std::vector<int> chain;
};

struct Config {
  int D = 64, R = 19, TA = 1, TL = 2;
};

// RD values for one kernel. ENTRY is -1.  RD(i, r) = max j < i with r in dst(j).
class KernelAnalysis {
 public:
  const Kernel& K;
  std::vector<int> lw;                                  // running last-writer per register
  std::vector<std::vector<std::pair<int, int>>> rd_at;  // rd_at[i] = {(r, RD(i, r))} queried
  explicit KernelAnalysis(const Kernel& k) : K(k) {}

  // O3: the reaching definition of register r at instruction i (linear order; predicated writes
  // count; back-edges are not followed) — P:446-448 "the previous SASS instruction executed by
  // the register".  Computed for all (i, r) pairs the later steps need, in one forward pass.
  void compute_rd(const std::vector<std::pair<int, int>>& queries) {
    rd_at.assign(K.ins.size(), {});
    for (auto& q : queries) rd_at[q.first].push_back({q.second, -1});
    lw.assign(320, -1);
    for (size_t i = 0; i < K.ins.size(); i++) {
      for (auto& q : rd_at[i]) q.second = lw[q.first];
      const Instr& I = K.ins[i];
      for (int dreg : {I.dst, I.dst2})
        if (dreg != kNoReg && !is_zero_reg(dreg))
          for (int w = 0; w < I.dst_w; w++) {
            int r = dreg + w;
            if ((is_ur(dreg) && r <= 318) || (!is_ur(dreg) && r <= 254)) lw[r] = (int)i;
          }
    }
  }
  int rd(int i, int r) const {
    for (auto& q : rd_at[i]) if (q.first == r) return q.second;
    fprintf(stderr, "oracle bug: RD(%d,%s) not computed\n", i, reg_name(r).c_str());
    abort();
  }
};

// O5 pointer operand of instruction J (the register the trace continues through).
// Returns 0: continue with *reg; 1: CONST terminal (*bank, *off); 2: IMM terminal.
int pointer_operand(const Instr& J, int* reg, int* bank, long long* off) {
  std::vector<const Opnd*> L;  // source operands after the dst, predicates skipped
  for (size_t k = (size_t)(J.dst_pos + 1); k < J.ops.size(); k++)
    if (J.ops[k].kind != K_PRED) L.push_back(&J.ops[k]);
  const Opnd* pick = nullptr;
  auto is_live_reg = [](const Opnd* o) { return o->kind == K_REG && !is_zero_reg(o->reg); };
  if ((J.op == "IMAD" || J.op == "UIMAD") && J.has_mod("WIDE")) {
    pick = L.size() > 2 ? L[2] : nullptr;
  } else if (J.op == "LEA" || J.op == "ULEA") {
    pick = L.size() > 1 ? L[1] : nullptr;
  } else if (J.op == "IADD3" || J.op == "UIADD3") {
    for (auto* o : L) if (o->kind == K_CREF) { pick = o; break; }
    if (!pick) for (auto* o : L) if (is_live_reg(o) && is_ur(o->reg)) { pick = o; break; }
    if (!pick) for (auto* o : L) if (is_live_reg(o) && !is_ur(o->reg)) { pick = o; break; }
  } else {
    for (auto* o : L) if (is_live_reg(o) || o->kind == K_CREF) { pick = o; break; }
  }
  if (pick && pick->kind == K_CREF) { *bank = pick->cbank; *off = pick->coff; return 1; }
  if (pick && is_live_reg(pick)) { *reg = pick->reg; return 0; }
  return 2;
}

// Collect every (i, r) RD query the trace from (i0, r0) can make (trace needs RD only along the
// chain, but the chain depends on RD values: we therefore compute RD for every instruction's
// pointer operand and for the starting registers; a plain superset).
void trace_queries(const Kernel& K, std::vector<std::pair<int, int>>& q) {
  for (size_t i = 0; i < K.ins.size(); i++) {
    const Instr& I = K.ins[i];
    if (I.dst != kNoReg) {
      int reg, bank;
      long long off;
      if (pointer_operand(I, &reg, &bank, &off) == 0) q.push_back({(int)i, reg});
    }
    if (I.mem >= 0 && I.ops[I.mem].base != kNoReg && !is_zero_reg(I.ops[I.mem].base))
      q.push_back({(int)i, I.ops[I.mem].base});
    for (int s : I.srcs) q.push_back({(int)i, s});
  }
}

// O5: the bounded backward trace of register r0 at instruction i (north_star).
Trace trace(const Kernel& K, const KernelAnalysis& A, int i, int r0, int D) {
  Trace T;
  if (r0 == kNoReg || is_zero_reg(r0)) { T.kind = T_IMM; return T; }
  int pos = i, r = r0;
  for (int step = 0; step < D; step++) {
    int j = A.rd(pos, r);                                   // 1. last writer
    if (j < 0) { T.kind = T_ENTRY; T.value = r; return T; }
    T.chain.push_back(j);                                   // 2. append
    pos = j;
    const Instr& J = K.ins[j];
    if (is_constload(J.op)) {                               // 3. constant bank load
      const Opnd* c = nullptr;
      for (size_t k = (size_t)(J.dst_pos + 1); k < J.ops.size(); k++)
        if (J.ops[k].kind == K_CREF) { c = &J.ops[k]; break; }
      long long off = (c ? c->coff : 0) + 4LL * (r - J.dst);
      int bank = c ? c->cbank : 0;
      if (bank == 0 && off >= K.param_base) { T.kind = T_PARAM; T.value = off; }
      else { T.kind = T_CONST; T.value = ((long long)bank << 32) | (off & 0xffffffffLL); }
      return T;
    }
    if (is_sreg(J.op)) { T.kind = T_SREG; T.value = j; return T; }      // 4.
    if (is_memload(J.op)) { T.kind = T_MEMORY; T.value = j; return T; }  // 5.
    int reg, bank;
    long long off;
    int pk = pointer_operand(J, &reg, &bank, &off);                       // 6.
    if (pk == 1) {
      if (bank == 0 && off >= K.param_base) { T.kind = T_PARAM; T.value = off; }
      else { T.kind = T_CONST; T.value = ((long long)bank << 32) | (off & 0xffffffffLL); }
      return T;
    }
    if (pk == 2) { T.kind = T_IMM; return T; }
    r = reg;
  }
  T.kind = T_TRUNC;
  return T;
}

std::string term_str(const Trace& T) {
  char b[64];
  switch (T.kind) {
    case T_NONE: return "NONE";
    case T_PARAM: snprintf(b, sizeof b, "PARAM:0x%llx", T.value); return b;
    case T_CONST: snprintf(b, sizeof b, "CONST:0x%llx:0x%llx", T.value >> 32, T.value & 0xffffffffLL); return b;
    case T_ENTRY: return "ENTRY:" + reg_name((int)T.value);
    case T_SREG: snprintf(b, sizeof b, "SREG:%lld", T.value); return b;
    case T_MEMORY: snprintf(b, sizeof b, "MEMORY:%lld", T.value); return b;
    case T_IMM: return "IMM";
    case T_TRUNC: return "TRUNC";
  }
  return "?";
}

// ---------------------------------------------------------------- sites
enum Rule { VEC = 0, SPILL, SHMEM, GATOM, RO, TEX, CONV, NRULES };
const char* kRuleName[NRULES] = {"VEC", "SPILL", "SHMEM", "GATOM", "RO", "TEX", "CONV"};

struct Site {
  int k = 0, idx = 0, rule = 0;
  int line = -1, loop_depth = 0;
  Trace tr;
  std::string attrs;
};

struct KernelStats {
  int gatom = 0, satom = 0, conv = 0, vec_already = 0, ustores = 0;
};

// Detection (the paper's dry run) over one kernel.
void detect_kernel(int kid, const Kernel& K, const Config& C, std::vector<Site>& sites, KernelStats& st) {
  const int n = (int)K.ins.size();
  KernelAnalysis A(K);
  std::vector<std::pair<int, int>> q;
  trace_queries(K, q);
  A.compute_rd(q);

  // O4 loop depth: number of backward BRA spans [t, pc(b)] containing pc(i).
  std::vector<int> loop_depth(n, 0);
  for (int b = 0; b < n; b++) {
    const Instr& B = K.ins[b];
    if (B.op != "BRA" || B.bra_target < 0) continue;
    long long t = B.bra_target;
    if (!(t < B.pc)) continue;  // forward or self branch
    for (int i = 0; i < n; i++)
      if (t <= K.ins[i].pc && K.ins[i].pc <= B.pc) loop_depth[i]++;
  }

  // O5 traces for every traced memory instruction (address base register).
  std::vector<Trace> tr(n);
  std::vector<bool> has_tr(n, false);
  for (int i = 0; i < n; i++) {
    const Instr& I = K.ins[i];
    if (!is_traced_memop(I.op) || I.mem < 0) continue;
    tr[i] = trace(K, A, i, I.ops[I.mem].base, C.D);
    has_tr[i] = true;
  }

  // global LDG key groups: key(i) = (base reg, RD(i, base))   [reading #3]
  struct Group {
    std::set<long long> off32, off_all;
    int n_loads = 0;
  };
  std::map<std::pair<int, int>, Group> groups;
  auto key_of = [&](int i) {
    int b = K.ins[i].ops[K.ins[i].mem].base;
    int rdv = (b == kNoReg || is_zero_reg(b)) ? -2 : A.rd(i, b);
    return std::make_pair(b, rdv);
  };
  for (int i = 0; i < n; i++) {
    const Instr& I = K.ins[i];
    if (I.op != "LDG" || I.mem < 0) continue;
    Group& g = groups[key_of(i)];
    g.n_loads++;
    g.off_all.insert(I.ops[I.mem].off);
    if (access_bits(I) == 32) g.off32.insert(I.ops[I.mem].off);
  }

  // n_arith(i) = |{ j in ARITH : exists source s of j with RD(j, s) = i }|
  std::vector<int> n_arith(n, 0);
  for (int j = 0; j < n; j++) {
    const Instr& J = K.ins[j];
    if (!is_arith(J)) continue;
    std::set<int> defs;
    for (int s : J.srcs) {
      int d = A.rd(j, s);
      if (d >= 0) defs.insert(d);
    }
    for (int d : defs) n_arith[d]++;
  }

  // O10 store roots of the kernel: resolved roots = PARAM offsets and ENTRY registers.
  std::set<std::pair<int, long long>> store_roots;
  for (int i = 0; i < n; i++) {
    if (!has_tr[i] || !is_store_class(K.ins[i].op)) continue;
    if (tr[i].kind == T_PARAM || tr[i].kind == T_ENTRY) store_roots.insert({tr[i].kind, tr[i].value});
    else st.ustores++;
  }

  for (int i = 0; i < n; i++) {
    const Instr& I = K.ins[i];
    auto emit = [&](int rule, const Trace& t, const std::string& attrs) {
      Site s;
      s.k = kid; s.idx = i; s.rule = rule; s.line = I.line; s.loop_depth = loop_depth[i];
      s.tr = t; s.attrs = attrs;
      sites.push_back(s);
    };
    char b[160];
    if (is_gatom(I.op)) st.gatom++;
    if (I.op == "ATOMS") st.satom++;
    if (is_conv(I.op)) st.conv++;
    if (I.op == "LDG" && I.mem >= 0) {
      int bits = access_bits(I);
      if (bits >= 64) st.vec_already++;  // "already vectorised" (64/128/256-bit)
      const Group& g = groups[key_of(i)];
      // O6 VEC: 32-bit LDG whose group has >= 2 distinct immediate offsets.
      if (bits == 32 && g.off32.size() >= 2) {
        long long mn = *g.off32.begin(), mx = *g.off32.rbegin();
        bool contig = true;
        long long prev = mn;
        for (auto it = std::next(g.off32.begin()); it != g.off32.end(); ++it) {
          if (*it - prev != 4) contig = false;
          prev = *it;
        }
        snprintf(b, sizeof b, "n=%zu min=%lld max=%lld contig=%d", g.off32.size(), mn, mx, contig ? 1 : 0);
        emit(VEC, tr[i], b);
      }
      // O8 SHMEM: arithmetic on the loaded value, loaded repeatedly or in a loop.
      if (n_arith[i] >= C.TA && (g.n_loads >= C.TL || loop_depth[i] >= 1)) {
        snprintf(b, sizeof b, "loads=%d arith=%d", g.n_loads, n_arith[i]);
        emit(SHMEM, tr[i], b);
      }
      // O10 RO: non-.CONSTANT load whose root no store of the kernel shares.
      bool ro = false;
      if (!I.has_mod("CONSTANT") && (tr[i].kind == T_PARAM || tr[i].kind == T_ENTRY))
        ro = store_roots.count({tr[i].kind, tr[i].value}) == 0;
      if (ro) emit(RO, tr[i], "");
      // O11 TEX: read-only and adjacent loads (any width) on the same base value.
      if (ro && g.off_all.size() >= 2) {
        snprintf(b, sizeof b, "n=%zu", g.off_all.size());
        emit(TEX, tr[i], b);
      }
    }
    // O7 SPILL: every STL / LDL; STL also names the last writer of the spilled register.
    if ((I.op == "STL" || I.op == "LDL") && I.mem >= 0) {
      std::string data = "-", cause = "-";
      if (I.op == "STL") {
        for (size_t k = (size_t)I.mem + 1; k < I.ops.size(); k++)
          if (I.ops[k].kind == K_REG) {
            data = reg_name(I.ops[k].reg);
            if (!is_zero_reg(I.ops[k].reg)) {
              int c = A.rd(i, I.ops[k].reg);
              cause = c < 0 ? "E" : std::to_string(c);
            }
            break;
          }
      } else if (I.dst != kNoReg) {
        data = reg_name(I.dst);
      }
      snprintf(b, sizeof b, "data=%s cause=%s", data.c_str(), cause.c_str());
      emit(SPILL, tr[i], b);
    }
    // O9 GATOM
    if (is_gatom(I.op) && I.mem >= 0) emit(GATOM, tr[i], "");
    // O12 CONV
    if (is_conv(I.op)) emit(CONV, Trace(), "");
  }
}

// ---------------------------------------------------------------- O16 register pressure
// "GPUscout presents the number of additional registers needed by each SASS instruction"
// (SURVEY §8f row 4). Live general-purpose registers per
// instruction by backward dataflow over the kernel's control-flow graph (reading R36):
//   live_in(i) = uses(i) ∪ (live_out(i) \ defs(i))   (a guarded instruction kills nothing)
//   live_out(i) = ∪ live_in(s), s ∈ succ(i)           (BRA target; fall-through unless an
//                                                      unguarded BRA / EXIT / RET)
//   count(i) = |live_in(i) ∪ defs(i)|, R1 (the stack pointer) counted live after its definition.
// Only R0..R254 (nvdisasm's "GPR #" column). additional(i) = count(i) - count(i-1).

// register width of a store / atomic data operand (R36, R38a/d): .256 -> 4 per data operand (two
// quads), .128 -> 4, STSM .4/.2 -> 4/2, STTM as LDTM, .64 or a 64-bit type -> 2
int data_width(const Instr& I) {
  for (auto& m : I.mods) if (m == "256" || m == "128") return 4;
  if (I.op == "STSM") return I.has_mod("4") ? 4 : (I.has_mod("2") ? 2 : 1);
  if (I.op == "STTM") return tmem_regs(I);
  for (auto& m : I.mods) if (m == "64" || is_64type(m)) return 2;
  return 1;
}

// GPR uses of instruction I, pair/quad registers expanded (R36, R38)
std::set<int> gpr_uses(const Instr& I) {
  std::set<int> u;
  int srcw = op_in(I.op, {"DADD", "DMUL", "DFMA", "DSETP", "DMNMX"}) ? 2 : 1;
  if (op_in(I.op, {"F2F", "I2F", "F2I", "I2I", "F2FP", "I2FP", "F2IP"})) srcw = conv_widths(I).second;  // R38e
  const bool store_like =
      op_in(I.op, {"STG", "STS", "STL", "ST", "RED", "REDG", "ATOMG", "ATOM", "ATOMS", "STSM", "STTM", "STAS"});
  const bool mma = I.op == "HMMA";
  const MmaRegs mr = mma ? mma_regs(I) : MmaRegs();
  // IMAD.HI adds a 64-bit addend: hi32(a * b + c:c+1) (R38h)
  const bool hi_add = I.op == "IMAD" && I.has_mod("HI");
  // an indirect branch / call / return reads a 64-bit target address (R38g)
  const bool target_pair = op_in(I.op, {"BRX", "BRXU", "JMX", "JMXU", "RET", "CALL"});
  const int last_dst = I.dst2_pos >= 0 ? I.dst2_pos : I.dst_pos;
  int last_mem = -1;  // .E ("extended" 64-bit global address) names the last memory operand (R38j)
  for (size_t k = 0; k < I.ops.size(); k++)
    if (I.ops[k].kind == K_MEM) last_mem = (int)k;
  int srcidx = 0;  // index among the non-predicate operands after the destination(s)
  for (size_t k = 0; k < I.ops.size(); k++) {
    if ((int)k == I.dst_pos || (int)k == I.dst2_pos) continue;
    const Opnd& o = I.ops[k];
    for (int r : o.regs) {
      if (r >= 255) continue;  // RZ, uniform registers
      int w = 1;
      // a memory base is a 64-bit pair when written Rb.64 (sm_100) or when the access is .E
      // ("extended", 64-bit addresses: sm_70's LDG.E [R8] reads R8:R9)
      if (o.kind == K_MEM) w = (r == o.base && (o.wide || (I.has_mod("E") && (int)k == last_mem))) ? 2 : 1;
      else if (o.kind == K_CREF) w = 1;
      else if (target_pair) w = 2;
      else if (store_like && k > 0) w = data_width(I);
      else if (mma) w = srcidx == 0 ? mr.a : (srcidx == 1 ? mr.b : mr.acc);
      else if (I.op == "IMAD" && I.has_mod("WIDE") && srcidx == 2) w = 2;
      else if (hi_add && srcidx == 2) w = 2;
      else w = srcw;
      for (int q = 0; q < w && r + q < 255; q++) u.insert(r + q);
    }
    if ((int)k > last_dst && o.kind != K_PRED) srcidx++;
  }
  if (I.op == "CALL") { u.insert(0); u.insert(1); }  // R38g: the call reads R0 and the stack pointer R1
  return u;
}

// R38g: registers a CALL may overwrite (the ABI's caller-saved GPRs, as nvdisasm's life ranges show
// them on sm_100a): R0, R3..R15 and R32+8j..R35+8j (j = 0..8), limited to the kernel's registers.
bool call_clobbered(int r) { return r == 0 || (r >= 3 && r <= 15) || (r >= 32 && r <= 99 && (r - 32) % 8 < 4); }

// GPR definitions of instruction I: the destination(s) and the registers their width covers (O2,
// R24, R38); a CALL defines its clobbered registers below `nregs` (the kernel's register count).
std::set<int> gpr_defs(const Instr& I, int nregs = 255) {
  std::set<int> d;
  for (int dreg : {I.dst, I.dst2})
    if (dreg != kNoReg && dreg < 255)
      for (int q = 0; q < I.dst_w && dreg + q < 255; q++) d.insert(dreg + q);
  if (I.op == "CALL")
    for (int r = 0; r < nregs && r < 255; r++)
      if (call_clobbered(r)) d.insert(r);
  return d;
}

// The kernel's register count (R38k): REG:N of the dump's cuobjdump -res-usage block when it has
// one, else one past the highest GPR any instruction reads or writes (widths expanded).
int kernel_nregs(const Kernel& K) {
  if (K.regcount > 0) return K.regcount;
  int m = 0;
  for (auto& I : K.ins) {
    for (int r : gpr_uses(I)) m = std::max(m, r + 1);
    for (int r : gpr_defs(I, 0)) m = std::max(m, r + 1);
  }
  return m;
}

std::vector<std::set<int>> live_sets(const Kernel& K) {
  const int n = (int)K.ins.size();
  std::vector<std::set<int>> use(n), def(n);
  std::vector<std::vector<int>> succ(n);
  int r1def = -1;
  const int nregs = kernel_nregs(K);
  for (int i = 0; i < n; i++) {
    const Instr& I = K.ins[i];
    use[i] = gpr_uses(I);
    def[i] = gpr_defs(I, nregs);
    if (r1def < 0 && def[i].count(1)) r1def = i;
    bool cond = I.guarded;
    // a branch with a predicate or register condition before its target (BRA.U !UP0, 0x..;
    // BRA.DIV UR4, 0x..) may fall through (R38i)
    if (I.op == "BRA")
      for (size_t k = 0; k + 1 < I.ops.size(); k++)
        cond |= (I.ops[k].kind == K_PRED && I.ops[k].pred_var) || I.ops[k].kind == K_REG;
    const bool branch = I.op == "BRA" && I.bra_target >= 0 && I.bra_target / 16 < n;
    if (branch) succ[i].push_back((int)(I.bra_target / 16));
    // an indirect branch continues at each of its listed targets (nvdisasm BRANCH_TARGETS, R38i)
    const bool brx = op_in(I.op, {"BRX", "BRXU", "JMX", "JMXU"});
    if (brx)
      for (long long t : I.brx_targets)
        if (t / 16 < n) succ[i].push_back((int)(t / 16));
    const bool ends = (I.op == "EXIT" || I.op == "RET" || branch || brx) && !cond;
    if (!ends && i + 1 < n) succ[i].push_back(i + 1);
  }
  // R38g: a RET hands the callee-saved registers (those a CALL does not clobber, below the kernel's
  // register count; R1 is counted separately) back to the caller: they are live out of it
  std::set<int> callee_saved;
  for (int r = 0; r < nregs && r < 255; r++)
    if (r != 1 && !call_clobbered(r)) callee_saved.insert(r);
  std::vector<std::set<int>> in(n);
  for (bool changed = true; changed;) {  // round-robin to the fixed point
    changed = false;
    for (int i = n - 1; i >= 0; i--) {
      std::set<int> out;
      for (int s : succ[i]) out.insert(in[s].begin(), in[s].end());
      if (K.ins[i].op == "RET") out.insert(callee_saved.begin(), callee_saved.end());
      std::set<int> li = use[i];
      for (int r : out)
        if (K.ins[i].guarded || !def[i].count(r)) li.insert(r);
      if (li != in[i]) { in[i] = li; changed = true; }
    }
  }
  std::vector<std::set<int>> live(n);
  for (int i = 0; i < n; i++) {
    live[i] = in[i];
    live[i].insert(def[i].begin(), def[i].end());
    if (r1def >= 0 && i > r1def) live[i].insert(1);
  }
  return live;
}

// count(i) = |live_in(i) ∪ defs(i)| (+ R1 after its definition)
std::vector<int> live_counts(const Kernel& K) {
  std::vector<int> cnt;
  for (auto& s : live_sets(K)) cnt.push_back((int)s.size());
  return cnt;
}

// ---------------------------------------------------------------- O13-O15
struct RawSample { uint32_t kernel, pc, reason; };
// pre-aggregated PC-sampling record (CUPTI CUpti_PCSamplingPCData shape: one (pc, stall reason)
// with its sample count, P:215-227 / SURVEY [probe 8]); `count` samples of that (kernel, pc, reason)
struct CountRec { uint32_t kernel, pc, reason, count; };

// The 19 ncu / CUPTI stall reasons in id order (R17, SURVEY [probe 9]); a CUPTI name is
// "smsp__pcsamp_warps_issue_stalled_<reason>[_not_issued]" (R39).
const char* kReasonName[19] = {"barrier", "branch_resolving", "dispatch_stall", "drain", "imc_miss",
                               "lg_throttle", "long_scoreboard", "math_pipe_throttle", "membar",
                               "mio_throttle", "misc", "no_instructions", "not_selected", "selected",
                               "short_scoreboard", "sleeping", "tex_throttle", "wait", "warpgroup_arrive"};

const int kRel[NRULES] = {
    // bit r set = reason r in REL(rule).  long_scoreboard = 6, lg_throttle = 5, tex_throttle = 16
    1 << 6,                 // VEC
    (1 << 6) | (1 << 5),    // SPILL P:616-624
    1 << 6,                 // SHMEM [R14 reading]
    1 << 5,                 // GATOM P:685-687
    1 << 6,                 // RO    [reading]
    (1 << 6) | (1 << 16),   // TEX
    -1,                     // CONV  all reasons [reading]
};

}  // namespace

int main(int argc, char** argv) {
  std::string sass_path, samples_path, counts_path, cupti_path, out_path, join = "pc";
  unsigned long long cupti_crc = 0;
  Config C;
  long long K_top = -1;
  int kbegin = 0, kend = -1;
  bool detect = true, hist = true, timing = false, quiet = false, liveness = false, no_hlines = false,
       regsets = false;
  for (int a = 1; a < argc; a++) {
    std::string s = argv[a];
    auto nxt = [&]() { return std::string(a + 1 < argc ? argv[++a] : ""); };
    if (s == "--sass") sass_path = nxt();
    else if (s == "--samples") samples_path = nxt();
    else if (s == "--counts") counts_path = nxt();  // CountRec records, added to the same histogram
    else if (s == "--cupti") cupti_path = nxt();    // CUPTI PC-sampling records (text form, R39)
    else if (s == "--cupti-crc") cupti_crc = strtoull(nxt().c_str(), nullptr, 0);  // 0: any module
    else if (s == "--join") join = nxt();            // pc (default) | line | consumer
    else if (s == "--out") out_path = nxt();
    else if (s == "--D") C.D = atoi(nxt().c_str());
    else if (s == "--R") C.R = atoi(nxt().c_str());
    else if (s == "--ta") C.TA = atoi(nxt().c_str());
    else if (s == "--tl") C.TL = atoi(nxt().c_str());
    else if (s == "--k") K_top = atoll(nxt().c_str());
    else if (s == "--kbegin") kbegin = atoi(nxt().c_str());
    else if (s == "--kend") kend = atoi(nxt().c_str());
    else if (s == "--no-detect") detect = false;
    else if (s == "--liveness") liveness = true;   // L lines: live GPRs per instruction (O16)
    else if (s == "--regsets") regsets = true;     // G lines: GPR defs and uses per instruction (O16 inputs)
    else if (s == "--no-hist") hist = false;
    else if (s == "--time") timing = true;
    else if (s == "--quiet") quiet = true;  // timing runs: compute everything, print only K/N lines
    else if (s == "--no-hlines") no_hlines = true;  // full-size runs: every line but the H lines
    else { fprintf(stderr, "unknown arg %s\n", s.c_str()); return 2; }
  }
  if (join != "pc" && join != "line" && join != "consumer") { fprintf(stderr, "unknown join %s\n", join.c_str()); return 2; }
  auto now = [] { return std::chrono::steady_clock::now(); };
  auto secs = [](auto a, auto b) { return std::chrono::duration<double>(b - a).count(); };
  FILE* f = fopen(sass_path.c_str(), "rb");
  if (!f) { fprintf(stderr, "cannot open %s\n", sass_path.c_str()); return 2; }
  std::string text;
  {
    fseek(f, 0, SEEK_END);
    long sz = ftell(f);
    fseek(f, 0, SEEK_SET);
    text.resize((size_t)sz);
    if (sz && fread(&text[0], 1, (size_t)sz, f) != (size_t)sz) return 2;
    fclose(f);
  }
  auto t0 = now();
  std::vector<Kernel> ks;
  try { ks = parse_sass(text); } catch (ParseError& e) { fprintf(stderr, "parse error: %s\n", e.msg.c_str()); return 3; }
  auto t1 = now();
  if (kend < 0 || kend > (int)ks.size()) kend = (int)ks.size();
  FILE* out = out_path.empty() ? stdout : fopen(out_path.c_str(), "wb");
  fprintf(out, "# gs-canonical v1\n");
  fprintf(out, "CFG D=%d R=%d TA=%d TL=%d\n", C.D, C.R, C.TA, C.TL);

  std::vector<Site> sites;
  std::vector<KernelStats> stats(ks.size());
  if (detect)
    for (int k = kbegin; k < kend; k++) detect_kernel(k, ks[k], C, sites, stats[k]);
  auto t2 = now();
  std::sort(sites.begin(), sites.end(), [](const Site& a, const Site& b) {
    if (a.k != b.k) return a.k < b.k;
    if (a.idx != b.idx) return a.idx < b.idx;
    return a.rule < b.rule;
  });
  if (detect) {
    for (int k = kbegin; k < kend; k++)
      fprintf(out, "K %d %zu %zu gatom=%d satom=%d conv=%d vec_already=%d ustores=%d name=%s\n", k,
              ks[k].ins.size(), ks[k].first_slot, stats[k].gatom, stats[k].satom, stats[k].conv,
              stats[k].vec_already, stats[k].ustores, ks[k].name.c_str());
    for (auto& s : sites) {
      if (quiet) break;
      std::string chain;
      for (size_t c = 0; c < s.tr.chain.size(); c++) chain += (c ? "," : "") + std::to_string(s.tr.chain[c]);
      if (chain.empty()) chain = "-";
      std::string line = s.line < 0 ? "-" : std::to_string(s.line);
      fprintf(out, "S %d %d %s line=%s ld=%d term=%s d=%zu chain=%s%s%s\n", s.k, s.idx, kRuleName[s.rule],
              line.c_str(), s.loop_depth, term_str(s.tr).c_str(), s.tr.chain.size(), chain.c_str(),
              s.attrs.empty() ? "" : " ", s.attrs.c_str());
    }
  }
  if (liveness)
    for (int k = kbegin; k < kend; k++) {
      std::vector<int> cnt = live_counts(ks[k]);
      for (size_t i = 0; i < cnt.size(); i++)
        fprintf(out, "L %d %zu %d %d\n", k, i, cnt[i], cnt[i] - (i ? cnt[i - 1] : 0));
    }
  if (regsets)  // the def / use / live sets of O16, one G line per instruction (test pins)
    for (int k = kbegin; k < kend; k++) {
      const int nregs = kernel_nregs(ks[k]);
      const std::vector<std::set<int>> live = live_sets(ks[k]);
      auto join = [](const std::set<int>& s) {
        std::string r;
        for (int x : s) r += (r.empty() ? "" : ",") + std::to_string(x);
        return r.empty() ? std::string("-") : r;
      };
      for (size_t i = 0; i < ks[k].ins.size(); i++)
        fprintf(out, "G %d %zu def=%s use=%s live=%s\n", k, i, join(gpr_defs(ks[k].ins[i], nregs)).c_str(),
                join(gpr_uses(ks[k].ins[i])).c_str(), join(live[i]).c_str());
    }
  if (hist && (!samples_path.empty() || !counts_path.empty() || !cupti_path.empty())) {
    // O13: H[slot][reason] += 1 for every valid sample.
    size_t P = 0;
    for (auto& k : ks) P += k.ins.size();
    std::vector<uint64_t> H(P * 32, 0);
    uint64_t N = 0, invalid = 0;
    auto valid = [&](uint32_t kernel, uint32_t pc, uint32_t reason) {
      return kernel < ks.size() && pc % 16 == 0 && pc / 16 < ks[kernel].ins.size() && reason < (uint32_t)C.R;
    };
    auto th0 = now();
    if (!samples_path.empty()) {
      FILE* sf = fopen(samples_path.c_str(), "rb");
      if (!sf) { fprintf(stderr, "cannot open %s\n", samples_path.c_str()); return 2; }
      std::vector<RawSample> buf(1 << 16);
      while (size_t got = fread(buf.data(), sizeof(RawSample), buf.size(), sf)) {
        for (size_t q = 0; q < got; q++) {
          const RawSample& s = buf[q];
          N++;
          if (!valid(s.kernel, s.pc, s.reason)) { invalid++; continue; }
          H[(ks[s.kernel].first_slot + s.pc / 16) * 32 + s.reason]++;
        }
      }
      fclose(sf);
    }
    if (!counts_path.empty()) {
      // pre-aggregated records: H[slot][reason] += count (the same histogram as `count` samples)
      FILE* cf = fopen(counts_path.c_str(), "rb");
      if (!cf) { fprintf(stderr, "cannot open %s\n", counts_path.c_str()); return 2; }
      CountRec r;
      while (fread(&r, sizeof r, 1, cf) == 1) {
        N += r.count;
        if (!valid(r.kernel, r.pc, r.reason)) { invalid += r.count; continue; }
        H[(ks[r.kernel].first_slot + r.pc / 16) * 32 + r.reason] += r.count;
      }
      fclose(cf);
    }
    uint64_t skipped = 0;
    if (!cupti_path.empty()) {
      // CUPTI PC sampling (§2.2; SURVEY [probe 8]; R39): one record per (function, pc
      // offset) with per-stall-reason sample counts; the stall-reason table maps CUPTI's indices to
      // names. Text form (tests write it from the same records the library reads):
      //   T <index> <name>                                        stall-reason table entry
      //   P <cubinCrc> <functionName> <pcOffset> <index>:<samples> ...   one CUpti_PCSamplingPCData
      // kernel = the kernel of the dump with that name; reason = the name's position in kReasonName
      // after the prefix; "_not_issued" counters are a subset of the same samples: skipped; a
      // foreign cubin (crc filter), unknown function or reason, or an invalid pc: invalid (R30).
      FILE* pf = fopen(cupti_path.c_str(), "rb");
      if (!pf) { fprintf(stderr, "cannot open %s\n", cupti_path.c_str()); return 2; }
      std::map<unsigned long long, std::string> table;
      std::map<std::string, int> kid;
      for (size_t k = 0; k < ks.size(); k++) kid.emplace(ks[k].name, (int)k);
      const std::string prefix = "smsp__pcsamp_warps_issue_stalled_", ni = "_not_issued";
      char lb[1 << 16];
      while (fgets(lb, sizeof lb, pf)) {
        std::vector<std::string> f;
        for (char* t = strtok(lb, " \t\r\n"); t; t = strtok(nullptr, " \t\r\n")) f.push_back(t);
        if (f.size() == 3 && f[0] == "T") { table[strtoull(f[1].c_str(), nullptr, 0)] = f[2]; continue; }
        if (f.size() < 4 || f[0] != "P") continue;
        const unsigned long long crc = strtoull(f[1].c_str(), nullptr, 0);
        const unsigned long long pc = strtoull(f[3].c_str(), nullptr, 0);
        auto ki = kid.find(f[2]);
        for (size_t q = 4; q < f.size(); q++) {
          const size_t c = f[q].find(':');
          const unsigned long long idx = strtoull(f[q].substr(0, c).c_str(), nullptr, 0);
          const unsigned long long cnt = strtoull(f[q].substr(c + 1).c_str(), nullptr, 0);
          std::string name = table.count(idx) ? table[idx] : std::string();
          if (name.size() > ni.size() && name.compare(name.size() - ni.size(), ni.size(), ni) == 0) {
            skipped += cnt;
            continue;
          }
          N += cnt;
          int reason = -1;
          if (name.compare(0, prefix.size(), prefix) == 0)
            for (int r = 0; r < 19; r++)
              if (name.substr(prefix.size()) == kReasonName[r]) reason = r;
          const bool ok = (cupti_crc == 0 || crc == cupti_crc) && ki != kid.end() && reason >= 0 &&
                          pc <= 0xffffffffull && valid((uint32_t)ki->second, (uint32_t)pc, (uint32_t)reason);
          if (!ok) { invalid += cnt; continue; }
          H[(ks[ki->second].first_slot + pc / 16) * 32 + reason] += cnt;
        }
      }
      fclose(pf);
    }
    auto th1 = now();
    uint64_t mass = 0;
    for (size_t b = 0; b < H.size(); b++)
      if (H[b]) {
        if (!quiet && !no_hlines) fprintf(out, "H %zu %zu %llu\n", b / 32, b % 32, (unsigned long long)H[b]);
        mass += H[b];
      }
    fprintf(out, "N total=%llu valid=%llu invalid=%llu\n", (unsigned long long)N, (unsigned long long)mass,
            (unsigned long long)invalid);
    if (!cupti_path.empty()) fprintf(out, "C skipped=%llu\n", (unsigned long long)skipped);  // _not_issued (R39)
    // O14 join: counts at the site's PC, site total, kernel total, REL sum.
    std::vector<uint64_t> ktot(ks.size(), 0);
    for (size_t k = 0; k < ks.size(); k++)
      for (size_t i = 0; i < ks[k].ins.size(); i++)
        for (int r = 0; r < 32; r++) ktot[k] += H[(ks[k].first_slot + i) * 32 + r];
    // The row a site is joined with (R18, R33): join=pc -> the site PC's row;
    // join=line -> the sum of the rows of every instruction of the kernel on the same source line
    // (file, line) as the site ("stall reasons ... at the line numbers identified"), or
    // the site PC's row when the site has no line information.
    // join=consumer (R37, [probe 9]: scoreboard stalls are sampled at the
    // instruction waiting for the data, not at its producer): the site PC's row plus the rows of
    // its direct consumers, the instructions j of the kernel that read a GPR (uses as in O16,
    // pairs expanded) whose last writer before j (linear order, predicated writes count, as O3)
    // is the site instruction. Each consumer counts once.
    std::map<int, std::vector<std::vector<int>>> consumers;
    auto consumers_of = [&](int k) -> const std::vector<std::vector<int>>& {
      auto it = consumers.find(k);
      if (it != consumers.end()) return it->second;
      const Kernel& K = ks[k];
      std::vector<std::vector<int>> cons(K.ins.size());
      std::vector<int> lw(255, -1);  // last writer of R0..R254 so far
      for (size_t j = 0; j < K.ins.size(); j++) {
        const Instr& J = K.ins[j];
        std::set<int> defs;
        for (int r : gpr_uses(J))
          if (lw[r] >= 0) defs.insert(lw[r]);
        for (int d : defs) cons[d].push_back((int)j);
        if (J.dst != kNoReg && J.dst < 255)
          for (int w = 0; w < J.dst_w && J.dst + w < 255; w++) lw[J.dst + w] = (int)j;
      }
      return consumers.emplace(k, std::move(cons)).first->second;
    };
    auto site_row = [&](const Site& s) {
      std::vector<uint64_t> row(32, 0);
      const Kernel& K = ks[s.k];
      const Instr& I = K.ins[s.idx];
      if (join == "consumer") {
        for (int r = 0; r < 32; r++) row[r] = H[(K.first_slot + s.idx) * 32 + r];
        for (int j : consumers_of(s.k)[s.idx])
          for (int r = 0; r < 32; r++) row[r] += H[(K.first_slot + j) * 32 + r];
        return row;
      }
      if (join == "pc" || I.line < 0) {
        for (int r = 0; r < 32; r++) row[r] = H[(K.first_slot + s.idx) * 32 + r];
        return row;
      }
      for (size_t i = 0; i < K.ins.size(); i++) {
        bool same = (int)i == s.idx;
        if (join == "line" && I.line >= 0) same = K.ins[i].line == I.line && K.ins[i].file == I.file;
        if (!same) continue;
        for (int r = 0; r < 32; r++) row[r] += H[(K.first_slot + i) * 32 + r];
      }
      return row;
    };
    struct Ranked { const Site* s; uint64_t rel, tot; std::vector<uint64_t> row; };
    std::vector<Ranked> rk;
    for (auto& s : sites) {
      std::vector<uint64_t> row = site_row(s);
      uint64_t tot = 0, rel = 0;
      for (int r = 0; r < 32; r++) {
        tot += row[r];
        if (kRel[s.rule] == -1 || (kRel[s.rule] >> r) & 1) rel += row[r];
      }
      rk.push_back({&s, rel, tot, row});
    }
    // O15 rank: (rel desc, tot desc, kernel asc, idx asc, rule asc)
    std::sort(rk.begin(), rk.end(), [](const Ranked& a, const Ranked& b) {
      if (a.rel != b.rel) return a.rel > b.rel;
      if (a.tot != b.tot) return a.tot > b.tot;
      if (a.s->k != b.s->k) return a.s->k < b.s->k;
      if (a.s->idx != b.s->idx) return a.s->idx < b.s->idx;
      return a.s->rule < b.s->rule;
    });
    size_t lim = K_top < 0 ? rk.size() : std::min(rk.size(), (size_t)K_top);
    auto tr1 = now();
    if (timing) fprintf(stderr, "TIME rank_s=%.6f sites=%zu\n", secs(th1, tr1), rk.size());
    for (size_t q = 0; q < lim && !quiet; q++) {
      const Site& s = *rk[q].s;
      std::string h;  // reported counts are 32-bit, saturating (R34)
      for (int r = 0; r < C.R; r++) h += (r ? "," : "") + std::to_string(std::min<uint64_t>(rk[q].row[r], 0xffffffffull));
      fprintf(out, "R %zu %d %d %s rel=%llu tot=%llu ktot=%llu h=%s\n", q, s.k, s.idx, kRuleName[s.rule],
              (unsigned long long)rk[q].rel, (unsigned long long)rk[q].tot, (unsigned long long)ktot[s.k], h.c_str());
    }
    if (timing) fprintf(stderr, "TIME hist_s=%.6f samples=%llu\n", secs(th0, th1), (unsigned long long)N);
  }
  auto t3 = now();
  if (timing)
    fprintf(stderr, "TIME parse_s=%.6f detect_s=%.6f total_s=%.6f instrs=%zu sites=%zu\n", secs(t0, t1),
            secs(t1, t2), secs(t0, t3), [&] { size_t n = 0; for (auto& k : ks) n += k.ins.size(); return n; }(),
            sites.size());
  if (out != stdout) fclose(out);
  return 0;
}
