"""Fold time of one preset at several record counts (fixed cost vs per-record cost):
    python tools/time_scale.py c2 15 1000000,2500000,5000000,10000000,20000000"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

name, mask = sys.argv[1], int(sys.argv[2])
sizes = [int(x) for x in sys.argv[3].split(",")]
P, _, _, _ = gen.preset(name)
s = torch.cuda.current_stream()
for lim in sizes:
    d = gen.generate_device(P, lim)
    ctx = sassi.Context(d["sites"], P.total_warps, mask)
    ts = []
    for it in range(7):
        ctx.reset(s)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        ctx.consume(d, stream=s)
        b.record(s)
        b.synchronize()
        if it >= 2:
            ts.append(a.elapsed_time(b))
    print("%s mask %d n %d: %.4f ms" % (name, mask, d["n"], sum(ts) / len(ts)), flush=True)
    ctx.close()
    del d
    torch.cuda.empty_cache()
