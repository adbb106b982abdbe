// loader.h — host SASS parser/packer interface (see loader.cpp).
#pragma once
#include <string>
#include <vector>

#include "record.h"

namespace gs {

struct ParsedKernel {
  std::string name;
  uint32_t param_base = 0x380;
  std::vector<Rec> recs;
  std::vector<int32_t> lines;  // source line per instruction, -1 if unknown
  std::vector<int32_t> lkeys;  // source-line key per instruction: kernel-local id of (file, line), -1 if unknown
  uint32_t n_lkeys = 0;
  // register-pressure inputs (R36): GPR uses per instruction (CSR, widths expanded) and branch
  // targets (kernel-local instruction index, -1 if none / unresolved)
  std::vector<uint32_t> use_off;  // n + 1
  std::vector<uint8_t> use_reg;
  std::vector<int32_t> tgt;       // -2 - x: indirect branch x with the successor list below (R38i)
  std::vector<uint32_t> xtgt_off; // indirect-branch successor lists (CSR over x; kernel-local indices)
  std::vector<int32_t> xtgt;
  uint32_t nregs = 0;             // the kernel's GPR count (R38k): REG:N of -res-usage, else max touched + 1
};

// Parses cuobjdump -sass / nvdisasm [-g] text into per-kernel packed records using up to n_threads threads.
// Returns false and sets *err ("line N: ...") on malformed input.
bool parse_sass(const char* text, size_t len, int n_threads, std::vector<ParsedKernel>* out, std::string* err);

}  // namespace gs
