"""Diagnostics for the online trace mode: time trace_fold per kernel at several segment sizes, and
the whole-kernel TRACE run, with CUDA events (usage: python tools/online_diag.py [kernel] [size])."""
import sys
import time

import torch

sys.path.insert(0, ".")
from paper_conf_isca_stephensonhlejn15_b200 import sassi  # noqa: E402

name = sys.argv[1] if len(sys.argv) > 1 else "vecadd"
size = int(sys.argv[2]) if len(sys.argv) > 2 else 0
ik = sassi.InstrumentedKernel(name, size)
ctx = ik.context(sassi.SASSI_H_EVERY)
s = torch.cuda.current_stream()


def ev(fn):
    a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    w0 = time.perf_counter()
    a.record(s)
    r = fn()
    b.record(s)
    b.synchronize()
    return a.elapsed_time(b), (time.perf_counter() - w0) * 1e3, r


for bps in (0, 64, 512):
    for serial in (False, True):
        for rep in range(3):
            ctx.reset(s)
            t, w, st = ev(lambda: ik.trace_fold(ctx, blocks_per_segment=bps, serial=serial, stream=s))
        print("bps %4d serial %d: %.2f ms (wall %.2f) segments %d records %d" % (
            bps, serial, t, w, st["segments"], st["n_records"]), flush=True)
