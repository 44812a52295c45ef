"""Per-warp timeline of one fold (development build with -DSASSI_TIMELINE, via SASSI_LIB):
entry, end of the prologue, end of the chunk loop, exit — printed as spreads over the warps."""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

name, mask = sys.argv[1], int(sys.argv[2])
if name == "c5s":
    P, _, _, _ = gen.preset("c5")
    d = gen.generate_device(P, None, 0, 16384)
else:
    P, lim, _, _ = gen.preset(name)
    d = gen.generate_device(P, lim)
ctx = sassi.Context(d["sites"], P.total_warps, mask)
s = torch.cuda.current_stream()
for _ in range(3):
    ctx.reset(s)
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record(s)
    ctx.consume(d, stream=s)
    b.record(s)
    b.synchronize()
print("%s: event %.4f ms" % (name, a.elapsed_time(b)))
buf = np.zeros(4 * 148 * 32 * 4, dtype=np.uint64)
lib = sassi.lib()
lib.sassi_debug_timeline.argtypes = [ctypes.c_void_p, ctypes.c_size_t]
assert lib.sassi_debug_timeline(buf.ctypes.data, buf.nbytes) == 0
t = buf.reshape(-1, 4)[: 148 * 32].astype(np.int64)
t0 = t[:, 0].min()
t = (t - t0) / 1000.0  # us
for k, nm in enumerate(["entry", "prologue done", "loop done", "exit"]):
    c = t[:, k]
    print("  %-14s min %8.2f  p50 %8.2f  p90 %8.2f  max %8.2f us" % (nm, c.min(), np.median(c),
                                                                   np.percentile(c, 90), c.max()))
ld = t[:, 2].reshape(148, 32)
print("  loop-done spread within a CTA (max - min): p50 %.2f  max %.2f us" %
      (np.median(ld.max(1) - ld.min(1)), (ld.max(1) - ld.min(1)).max()))
print("  CTA loop-done max: min %.2f p50 %.2f max %.2f us" % (ld.max(1).min(), np.median(ld.max(1)), ld.max(1).max()))
print("  busy fraction (sum of warp loop time / (nwarps * last loop done)): %.3f" %
      ((t[:, 2] - t[:, 1]).sum() / (len(t) * t[:, 2].max())))
ctx.close()
