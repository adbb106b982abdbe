"""Canonical text report of a GPU run (the paper's text report, in the line format of
DESIGN.md §5). Product-side formatting of the library's outputs; it does not import oracle/."""
from __future__ import annotations

import numpy as np

from .binding import RULES

_KIND = ["NONE", "PARAM", "CONST", "ENTRY", "SREG", "MEMORY", "IMM", "TRUNC"]


def reg_name(r: int) -> str:
    if r == 511:
        return "-"
    if r < 256:
        return "RZ" if r == 255 else f"R{r}"
    return "URZ" if r == 319 else f"UR{r - 256}"


def term_str(kind: int, value: int) -> str:
    k = _KIND[kind]
    if k == "PARAM":
        return f"PARAM:{value:#x}"
    if k == "CONST":
        return f"CONST:{value >> 16:#x}:{value & 0xFFFF:#x}"
    if k == "ENTRY":
        return "ENTRY:" + reg_name(value)
    if k in ("SREG", "MEMORY"):
        return f"{k}:{value}"
    return k


def site_lines(sites: np.ndarray, chain: np.ndarray, lines: np.ndarray, first_slot: np.ndarray) -> list[str]:
    out = []
    for s in sites:
        rule = RULES[s["rule"]]
        d = int(s["depth"])
        off = int(s["chain_off"])
        ch = ",".join(str(int(x)) for x in chain[off:off + d]) if d else "-"
        ln = int(lines[int(first_slot[s["kernel"]]) + int(s["idx"])]) if len(lines) else -1
        line = "-" if ln < 0 else str(ln)
        a0, a1, a2 = int(s["a0"]), int(s["a1"]), int(s["a2"])
        if rule == "VEC":
            attrs = f" n={a0 & 0x3FFFFFFF} min={a1} max={a2} contig={(a0 >> 30) & 1}"
        elif rule == "SPILL":
            cause = "E" if a1 == -1 else ("-" if a1 == -2 else str(a1))
            attrs = f" data={reg_name(a0)} cause={cause}"
        elif rule == "SHMEM":
            attrs = f" loads={a0} arith={a1}"
        elif rule == "TEX":
            attrs = f" n={a0}"
        else:
            attrs = ""
        out.append(f"S {int(s['kernel'])} {int(s['idx'])} {rule} line={line} ld={int(s['loop_depth'])} "
                   f"term={term_str(int(s['term_kind']), int(s['term_value']))} d={d} chain={ch}{attrs}")
    return out


def canonical(ctx, k_begin: int = 0, k_end: int | None = None, hist=None, n_samples: int | None = None,
              n_invalid: int | None = None, ranked: np.ndarray | None = None, cfg_line: bool = True) -> str:
    """Canonical text of the last gs_detect (+ histogram and ranking when given)."""
    k_end = ctx.n_kernels if k_end is None else k_end
    first, n = ctx.kernel_table()
    out = ["# gs-canonical v1"]
    if cfg_line:
        out.append(f"CFG D={ctx.trace_depth} R={ctx.n_reasons} TA={ctx.cfg.shmem_min_arith} "
                   f"TL={ctx.cfg.shmem_min_loads}")
    ks = ctx.kernel_stats()
    for k in range(k_begin, k_end):
        st = ks[k]
        out.append(f"K {k} {int(n[k])} {int(first[k])} gatom={st['n_gatom']} satom={st['n_satom']} "
                   f"conv={st['n_conv']} vec_already={st['n_vec_already']} ustores={st['n_unresolved_stores']} "
                   f"name={ctx.kernel_name(k)}")
    sites, chain = ctx.sites()
    out += site_lines(sites, chain, ctx.instr_lines(), first)
    if hist is not None:
        row = getattr(ctx, "hist_row", 32)
        h = hist.detach().cpu().numpy() if hasattr(hist, "detach") else np.asarray(hist)
        h = h.astype(np.int64).reshape(-1, row)
        nzs, nzr = np.nonzero(h)
        out += [f"H {s} {r} {h[s, r]}" for s, r in zip(nzs, nzr)]
        valid = int(h.sum())
        out.append(f"N total={n_samples} valid={valid} invalid={n_invalid}")
        if ranked is not None:
            R = ctx.n_reasons
            for q, row in enumerate(ranked):
                hh = ",".join(str(int(x)) for x in row["counts"][:R])
                out.append(f"R {q} {int(row['kernel'])} {int(row['idx'])} {RULES[row['rule']]} rel={int(row['rel'])} "
                           f"tot={int(row['tot'])} ktot={int(row['ktot'])} h={hh}")
    return "\n".join(out) + "\n"
