"""Small workload for compute-sanitizer (memcheck / racecheck / synccheck / initcheck): T0 under
every handler set, a random edge trace, c1, the four instrumented kernels in every mode (inline,
trace, null ABI, injection), sampling and a 1-rank merge. Exits non-zero on any mismatch."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import t0_trace as T0  # noqa: E402
from gpu_helpers import to_device, gpu_table  # noqa: E402
from test_oracle import random_trace  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

s = T0.sites()
hdr, addr, val = T0.records()
d = to_device(s, hdr, addr, val)
for mask in (1, 2, 4, 8, 15, 16, 31):
    t = gpu_table(s, T0.N_WARPS, mask, d)
    assert np.array_equal(t, oracle.run(s, T0.N_WARPS, mask, hdr, addr, val)), mask
s2, W, h2, a2, v2 = random_trace(4321, n=3000)
t = gpu_table(s2, W, 31, to_device(s2, h2, a2, v2))
assert np.array_equal(t, oracle.run(s2, W, 31, h2, a2, v2))
t = gpu_table(s2, W, 31, to_device(s2, h2, a2, v2), pcs=[int(s2[1]["pc"]), int(s2[7]["pc"])])
assert np.array_equal(t, oracle.run(s2, W, 31, h2, a2, v2, pcs=[1, 7]))
P, lim, mask, _ = gen.preset("c1")
dc = gen.generate_device(P, lim)
ctx = sassi.Context(dc["sites"], P.total_warps, 31)
ctx.consume(dc)
ctx.sample(50, 7)
ctx.close()
for name, size in (("vecadd", 12800), ("bfs", 4096), ("sgemm", 32), ("stencil", 64)):
    ik = sassi.InstrumentedKernel(name, size)
    ctx = ik.context(sassi.SASSI_H_EVERY)
    for mode in (0, 1, 2, 4, 8, 16, 15, 31, sassi.SASSI_IK_NULL_ABI):
        ctx.reset()
        ik.run(mode, ctx if mode & 31 else None)
    ik.trace(ctx)
    ctx.close()
    ik.injection_campaign(k=20, seed=3)
    ik.close()
torch.cuda.synchronize()
print("sanitize workload ok")
