"""Dynamic sites at scale: fold the c4 stream (10^8 header records) with (a) every site registered
(the usual fold), (b) an empty site table and the insert-on-miss table on (the discovery pass:
every record goes to the dynamic table). CUDA events, median of 5. usage: python tools/dyn_bench.py"""
import statistics
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

P, lim, mask, _ = gen.preset("c4")
d = gen.generate_device(P, lim)
n = d["n"]
s = torch.cuda.current_stream()


def timed(ctx, rec, reps=6):
    ts = []
    for r in range(reps):
        ctx.reset(s)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        ctx.consume(rec, stream=s)
        b.record(s)
        b.synchronize()
        if r:
            ts.append(a.elapsed_time(b))
    return statistics.median(ts)


ctx = sassi.Context(d["sites"], P.total_warps, sassi.SASSI_H_INSTCOUNT)
t_reg = timed(ctx, d)
ctx.close()
empty = np.zeros(0, dtype=sassi.SITE_DTYPE)
hdr_only = dict(hdr=d["hdr"], addr=d["addr"][:0], val=d["val"][:0], chunk_base=d["chunk_base"], n=n,
                n_addr_rows=0, n_val_rows=0)
ctx = sassi.Context(empty, P.total_warps, sassi.SASSI_H_INSTCOUNT)
ctx.enable_dynamic_pcs(4096)
t_dyn = timed(ctx, hdr_only)
dyn, dropped = ctx.read_dynamic_pcs()
ctx.close()
print("registered sites: %.3f ms (%.2e rec/s); discovery pass: %.3f ms (%.2e rec/s), %d pcs, %d dropped, "
      "sum %d == n %d" % (t_reg, n / t_reg * 1e3, t_dyn, n / t_dyn * 1e3, len(dyn), dropped,
                          int(dyn["warp_execs"].sum()) + dropped, n))
