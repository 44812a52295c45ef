"""Oracle-side report formulas over a table image — test infrastructure only.

Each function restates a summary the paper prints (PAPER.md = /root/reference/PAPER.md):
  - value_profile_lines : the per-instruction dump of §7.2 (L601-L609)
  - table1_percent      : Table 1 static/dynamic divergent-branch % (L255-L271, L281)
  - fig7_pmf            : Fig.7 PMF over unique 32 B lines, thread-weighted (L373)
  - table2_percent      : Table 2 constant-bit / scalar %, static and dynamic (L577-L593, L613)
  - instmix_report      : Fig.3's dynamic_instr_counts[7] by category, with % of executed (L193-L199)
"""
from __future__ import annotations

import numpy as np

from . import IMIX_NAMES, sections


def value_profile_lines(table, sites, n_warps):
    """§7.2 dump (L601-L609): for each instruction that wrote registers, one line per destination
    ``R<n>[*] <- [b31..b0]`` with '1' = bit always one, '0' = always zero, 'T' = toggled, and '*'
    after the register name when every warp wrote one value across its lanes (scalar, L609)."""
    sec = sections(table, len(sites), n_warps)
    out = []
    for s, site in enumerate(sites):
        if int(sec["val"][s, 0]) == 0:
            continue
        lines = []
        for d in range(int(site["n_gpr_dst"])):
            ones, zeros = int(sec["ones"][s, d]), int(sec["zeros"][s, d])
            chars = []
            for b in range(31, -1, -1):
                if (ones >> b) & 1:
                    chars.append("1")
                elif (zeros >> b) & 1:
                    chars.append("0")
                else:
                    chars.append("T")
            star = "*" if int(sec["scalar"][s, d]) == 1 else ""
            lines.append("R%d%s <- [%s]" % (int(site["reg_num"][d]), star, "".join(chars)))
        out.append((int(site["pc"]), lines))
    return out


def table1_percent(br_stats):
    """Table 1 (L281): static % = divergent branch PCs / executed branch PCs; dynamic % =
    divergent warp-level branch executions / all warp-level branch executions.
    br_stats: array [S,5] (total, active, taken, nottaken, divergent)."""
    br = np.asarray(br_stats, dtype=np.float64)
    executed = br[:, 0] > 0
    n_static = int(executed.sum())
    n_static_div = int((br[:, 4][executed] > 0).sum())
    static = 100.0 * n_static_div / n_static if n_static else 0.0
    tot = br[:, 0].sum()
    dynamic = 100.0 * br[:, 4].sum() / tot if tot else 0.0
    return n_static, n_static_div, static, int(tot), int(br[:, 4].sum()), dynamic


def fig7_pmf(h32):
    """Fig.7 (L373): fraction of THREAD-level memory accesses issued from warps requesting N unique
    lines, N = 1..32 — each matrix cell [a-1][N-1] weighted by its active-thread count a."""
    h = np.asarray(h32, dtype=np.float64).reshape(32, 32)
    w = h * np.arange(1, 33, dtype=np.float64)[:, None]
    tot = w.sum()
    return w.sum(axis=0) / tot if tot else np.zeros(32)


def table2_percent(table, sites, n_warps):
    """Table 2 (L613): % of register bits that are constant and % of register writes that are
    scalar. Static weighs each (instruction, destination) equally; dynamic weighs it by its
    execution frequency (thread executions, the paper's `weight`, L555)."""
    sec = sections(table, len(sites), n_warps)
    cb_s = cb_d = sc_s = sc_d = 0.0
    n_s = w_d = 0.0
    for s, site in enumerate(sites):
        if int(sec["val"][s, 0]) == 0:
            continue
        w = float(sec["val"][s, 1])
        for d in range(int(site["n_gpr_dst"])):
            const = bin((int(sec["ones"][s, d]) | int(sec["zeros"][s, d])) & 0xFFFFFFFF).count("1")
            scalar = 1.0 if int(sec["scalar"][s, d]) == 1 else 0.0
            cb_s += const / 32.0
            sc_s += scalar
            n_s += 1
            cb_d += w * const / 32.0
            sc_d += w * scalar
            w_d += w
    if n_s == 0:
        return 0.0, 0.0, 0.0, 0.0
    return 100 * cb_d / w_d, 100 * sc_d / w_d, 100 * cb_s / n_s, 100 * sc_s / n_s


def instmix_report(table, n_sites, n_warps):
    """Fig.3 (L193-L199): the seven thread-level counters [memory, extended memory, controlxfer,
    sync, numeric, texture, total executed] as (name, count, % of total executed); categories
    overlap, so the percentages need not sum to 100."""
    imix = [int(x) for x in sections(table, n_sites, n_warps)["imix"][:7]]
    tot = imix[6]
    return [(n, c, 100.0 * c / tot if tot else 0.0) for n, c in zip(IMIX_NAMES, imix)]
