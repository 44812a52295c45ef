"""Host-side reports over a table image (what the paper's tools print from the handlers' counters).

PAPER.md = /root/reference/PAPER.md. Each function restates one of the paper's summaries:
  branch_table1      Table 1 (L255-L271, definitions): static / dynamic divergent-branch %
  branch_profile     Fig.5 (L333-L337): per-branch statistics sorted by dynamic branch count
  memdiv_pmf         Fig.7 (L373): PMF of unique 32 B lines per warp access, thread-weighted
  memdiv_heatmap     Fig.8 (L545): the 32x32 matrix normalised by its total
  value_dump         §7.2 (L601-L609): "R12 <- [000...TTT]" lines, '*' marks scalar registers
  value_table2       Table 2 (L577-L593, L613): constant-bit % and scalar %, static and dynamic
  instruction_mix    Fig.3 (L193-L199): the seven dynamic_instr_counts with % of executed
  injection_outcomes Fig.10 (L637-L667): % of injection runs per outcome
Independent of the test oracle (tests compare the two).
"""
from __future__ import annotations

import numpy as np

from . import sassi

MIX_NAMES = ("memory", "extended memory", "controlxfer", "sync", "numeric", "texture",
             "total executed")


def _sec(table, n_sites, n_warps):
    L = sassi.sassi_table_layout(n_sites, n_warps)
    S, t = int(n_sites), np.asarray(table, dtype=np.uint64)
    return {"br": t[L["br"]:L["mem"]].reshape(S, 5), "val": t[L["val"]:L["ones"]].reshape(S, 2),
            "ones": t[L["ones"]:L["zeros"]].reshape(S, 4),
            "zeros": t[L["zeros"]:L["scalar"]].reshape(S, 4),
            "scalar": t[L["scalar"]:L["h32"]].reshape(S, 4),
            "h32": t[L["h32"]:L["h128"]].reshape(32, 32), "imix": t[L["imix"]:L["pcsel"]],
            "pcmat": t[L["pcmat"]:L["total"]].reshape(4, 32, 32)}


def branch_table1(table, sites, n_warps):
    """(static branches executed, static divergent, static %, dynamic branches, dynamic divergent,
    dynamic %): a branch is statically divergent if any of its executions diverged (L281)."""
    br = _sec(table, len(sites), n_warps)["br"]
    total, div = br[:, 0].astype(np.int64), br[:, 4].astype(np.int64)
    seen = total > 0
    n, nd = int(seen.sum()), int((div[seen] > 0).sum())
    T, D = int(total.sum()), int(div.sum())
    return n, nd, (100.0 * nd / n if n else 0.0), T, D, (100.0 * D / T if T else 0.0)


def branch_profile(table, sites, n_warps):
    """Fig.5: one row per executed branch, most executed first:
    (pc, executions, divergent executions, active threads, taken threads, not-taken threads)."""
    br = _sec(table, len(sites), n_warps)["br"]
    rows = [(int(sites[i]["pc"]), int(b[0]), int(b[4]), int(b[1]), int(b[2]), int(b[3]))
            for i, b in enumerate(br) if b[0] > 0]
    return sorted(rows, key=lambda r: (-r[1], r[0]))


def memdiv_pmf(h32):
    """Fig.7: fraction of thread-level accesses issued by warps touching N unique lines (N=1..32);
    cell [a-1][N-1] carries a threads per warp access (L373)."""
    h = np.asarray(h32, dtype=np.float64).reshape(32, 32)
    per_n = (h * np.arange(1, 33)[:, None]).sum(axis=0)
    tot = per_n.sum()
    return per_n / tot if tot else per_n


def memdiv_heatmap(h32):
    """Fig.8: the (active threads x unique lines) matrix as fractions of all warp accesses."""
    h = np.asarray(h32, dtype=np.float64).reshape(32, 32)
    tot = h.sum()
    return h / tot if tot else h


def value_dump(table, sites, n_warps):
    """§7.2: {pc: ["R<n>[*] <- [b31..b0]", ...]} for every instruction that wrote registers;
    '1' / '0' = bit always one / zero, 'T' = toggled, '*' = scalar write (L603-L609)."""
    sec = _sec(table, len(sites), n_warps)
    out = {}
    for i, st in enumerate(sites):
        if sec["val"][i, 0] == 0:
            continue
        lines = []
        for d in range(int(st["n_gpr_dst"])):
            one, zero = int(sec["ones"][i, d]) & 0xFFFFFFFF, int(sec["zeros"][i, d]) & 0xFFFFFFFF
            bits = "".join("1" if one >> b & 1 else ("0" if zero >> b & 1 else "T")
                           for b in range(31, -1, -1))
            mark = "*" if int(sec["scalar"][i, d]) else ""
            lines.append("R%d%s <- [%s]" % (int(st["reg_num"][d]), mark, bits))
        out[int(st["pc"])] = lines
    return out


def value_table2(table, sites, n_warps):
    """Table 2 (L613): (dynamic constant-bit %, dynamic scalar %, static constant-bit %, static
    scalar %). Static weighs every written (instruction, destination) once; dynamic weighs it by
    the instruction's thread executions (the handler's `weight`, L555)."""
    sec = _sec(table, len(sites), n_warps)
    cs, ss, ws, cd, sd, wd = 0.0, 0.0, 0, 0.0, 0.0, 0.0
    for i, st in enumerate(sites):
        if sec["val"][i, 0] == 0:
            continue
        w = float(sec["val"][i, 1])
        for d in range(int(st["n_gpr_dst"])):
            frac = bin((int(sec["ones"][i, d]) | int(sec["zeros"][i, d])) & 0xFFFFFFFF).count("1") / 32.0
            sc = float(int(sec["scalar"][i, d]) != 0)
            cs, ss, ws = cs + frac, ss + sc, ws + 1
            cd, sd, wd = cd + w * frac, sd + w * sc, wd + w
    if not ws:
        return 0.0, 0.0, 0.0, 0.0
    return 100.0 * cd / wd, 100.0 * sd / wd, 100.0 * cs / ws, 100.0 * ss / ws


def instruction_mix(table, n_sites, n_warps):
    """Fig.3: [(category, thread-level count, % of total executed)] (categories overlap)."""
    m = [int(x) for x in _sec(table, n_sites, n_warps)["imix"][:7]]
    return [(name, c, 100.0 * c / m[6] if m[6] else 0.0) for name, c in zip(MIX_NAMES, m)]


def injection_outcomes(outcomes):
    """Fig.10: {outcome name: % of runs} from sassi_ik_inject results."""
    oc = np.asarray(outcomes["outcome"])
    n = max(len(oc), 1)
    return {name: 100.0 * float((oc == code).sum()) / n
            for code, name in enumerate(sassi.INJ_OUTCOME_NAMES)}
