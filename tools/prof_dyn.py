"""Discovery pass over c4's headers (empty site table, dynamic pcs on) for ncu."""
import sys

import numpy as np
import torch

sys.path.insert(0, ".")
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

P, lim, _, _ = gen.preset("c4")
d = gen.generate_device(P, lim)
rec = dict(hdr=d["hdr"], addr=d["addr"][:0], val=d["val"][:0], chunk_base=d["chunk_base"], n=d["n"],
           n_addr_rows=0, n_val_rows=0)
ctx = sassi.Context(np.zeros(0, dtype=sassi.SITE_DTYPE), P.total_warps, sassi.SASSI_H_INSTCOUNT)
ctx.enable_dynamic_pcs(4096)
for _ in range(2):
    ctx.reset()
    ctx.consume(rec)
torch.cuda.synchronize()
