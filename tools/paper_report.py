"""The paper's printed summaries from the GPU tables of the synthetic configs (c2 BFS-shaped, c3
SGEMM/stencil-shaped): Table 1 (branch divergence), Fig.7 (unique 32 B sectors per warp access,
thread-weighted), Table 2 (constant bits / scalar, dynamic and static), Fig.3 (instruction mix).
usage: python tools/paper_report.py OUT.md  (GPU; every table folded by sassi_consume)"""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_isca_stephensonhlejn15_b200 import gen, reports, sassi  # noqa: E402

out = ["# The paper's summaries on the synthetic workloads (B200, `tools/paper_report.py`)", "",
       "Every table below is computed by `reports.py` from a table image the CUDA fold produced "
       "(all five handlers). The workloads are synthetic (DESIGN.md §5): these are the formats of "
       "the paper's Table 1 / Fig.7 / Table 2 / Fig.3, not its applications' values.", ""]
for name, lim in (("c2", 10_000_000), ("c3", 20_000_000)):
    P, _, _, desc = gen.preset(name)
    d = gen.generate_device(P, lim)
    ctx = sassi.Context(d["sites"], P.total_warps, sassi.SASSI_H_EVERY)
    ctx.consume(d)
    t = ctx.read_tables()
    ctx.close()
    S, W, sites = len(d["sites"]), P.total_warps, d["sites"]
    n, nd, sp, T, D, dp = reports.branch_table1(t, sites, W)
    out += ["## %s (first %d records): %s" % (name, d["n"], desc), "",
            "Table 1 (L255-L271): static %d branches, %d divergent (%.0f %%); dynamic %d, %d divergent "
            "(%.1f %%)." % (n, nd, sp, T, D, dp), ""]
    lay = sassi.sassi_table_layout(S, W)
    h32 = t[lay["h32"]:lay["h128"]].reshape(32, 32)
    pmf = reports.memdiv_pmf(h32)
    out += ["Fig.7 (L373): thread-weighted share of accesses by unique 32 B sectors per warp access:", "",
            "| sectors | " + " | ".join(str(k) for k in (1, 2, 4, 8, 16, 32)) + " |",
            "|---|" + "---|" * 6,
            "| share | " + " | ".join("%.3f" % pmf[k - 1] for k in (1, 2, 4, 8, 16, 32)) + " |", ""]
    cd, sd, cs, ss = reports.value_table2(t, sites, W)
    out += ["Table 2 (L577-L593): constant bits %.0f %% / scalar %.0f %% (dynamic); %.0f %% / %.0f %% "
            "(static)." % (cd, sd, cs, ss), ""]
    mix = reports.instruction_mix(t, S, W)
    out += ["Fig.3 (L193-L199): " + ", ".join("%s %.1f %%" % (nm, pct) for nm, c, pct in mix), ""]
open(sys.argv[1], "w").write("\n".join(out) + "\n")
print("\n".join(out))
