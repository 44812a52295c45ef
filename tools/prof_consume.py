"""Profiling driver: generate a workload on cuda:0 and run sassi_consume `reps` times (for ncu)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c3"
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 3
mask = int(sys.argv[3]) if len(sys.argv) > 3 else gen.PRESETS[name][2]
P, lim, _, _ = gen.preset(name)
# c5 (8 shards, ~680 GB) is profiled on one shard of 16,384 warps, as the bench folds it
d = gen.generate_device(P, None, 0, 16384) if name == "c5" else gen.generate_device(P, lim)
ctx = sassi.Context(d["sites"], P.total_warps, mask)
for _ in range(reps):
    ctx.reset()
    ctx.consume(d)
torch.cuda.synchronize()
print("ok", d["n"])
