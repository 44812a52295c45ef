import sys; sys.path.insert(0, "."); sys.path.insert(0, "tests")
import numpy as np
import oracle
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi
for name, size in (("vecadd", 1 << 16), ("stencil", 64)):
    ik = sassi.InstrumentedKernel(name, size)
    ctx = ik.context(31)
    outs = []
    for _ in range(2):
        rec = ik.trace(ctx)
        h = gen.to_host(rec)
        outs.append(oracle.run(h["sites"], ik.n_warps, 31, h["hdr"], h["addr"], h["val"]))
    ctx.reset()
    ik.trace_fold(ctx, blocks_per_segment=0, serial=True)
    t = ctx.read_tables()
    print(name, "two traces equal:", np.array_equal(outs[0], outs[1]), " online == trace1:", np.array_equal(t, outs[0]), " online == trace2:", np.array_equal(t, outs[1]))
