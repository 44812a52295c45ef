"""Time the fold of one workload under several handler masks (CUDA events, mean of 5 after 2 warm-ups)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "c3"
masks = [int(m) for m in sys.argv[2].split(",")] if len(sys.argv) > 2 else [15, 4, 2, 1, 8, 9, 11, 13, 6]
if name == "c5s":  # one c5 warp shard (16,384 of the 131,072 warps, as bench.py folds them)
    P, _, _, _ = gen.preset("c5")
    d = gen.generate_device(P, None, 0, 16384)
else:
    P, lim, _, _ = gen.preset(name)
    d = gen.generate_device(P, lim)
s = torch.cuda.current_stream()
for m in masks:
    ctx = sassi.Context(d["sites"], P.total_warps, m)
    for _ in range(2):
        ctx.reset(s)
        ctx.consume(d, stream=s)
    ts = []
    for _ in range(5):
        ctx.reset(s)
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record(s)
        ctx.consume(d, stream=s)
        b.record(s)
        b.synchronize()
        ts.append(a.elapsed_time(b))
    print("%s mask %2d: %.3f ms" % (name, m, sum(ts) / len(ts)), flush=True)
    ctx.close()
