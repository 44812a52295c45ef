"""Randomised fuzz of the instrumented kernels (GPU): random problem sizes, handler modes (default
and SMEM), online-trace segment sizes; the inline tables, the fold of the kernel's whole trace and
the online trace fold must all equal the oracle on that trace (inline: but the record diagnostics).
usage: python tools/fuzz_inline.py [N_CASES] [SEED]"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle  # noqa: E402
from gpu_helpers import diff_tables  # noqa: E402
from paper_conf_isca_stephensonhlejn15_b200 import gen, sassi  # noqa: E402

n_cases = int(sys.argv[1]) if len(sys.argv) > 1 else 40
rng = np.random.default_rng(int(sys.argv[2]) if len(sys.argv) > 2 else 3)
fails = 0
for case in range(n_cases):
    name = str(rng.choice(["vecadd", "bfs", "sgemm", "stencil"]))
    size = {"vecadd": int(rng.integers(1, 1 << 18)), "bfs": int(rng.integers(1, 8192)),
            "sgemm": 16 * int(rng.integers(1, 9)), "stencil": 32 * int(rng.integers(1, 9))}[name]
    mask = int(rng.choice([1, 2, 4, 8, 15, 16, 31]))
    smem = int(rng.choice([0, sassi.SASSI_IK_SMEM]))
    seed = int(rng.integers(0, 2**31))
    ik = sassi.InstrumentedKernel(name, size, seed=seed)
    S, W = len(ik.sites), ik.n_warps
    ctx = ik.context(mask)
    rec = ik.trace(ctx)
    h = gen.to_host(rec)
    want = oracle.run(h["sites"], W, mask, h["hdr"], h["addr"], h["val"])
    msgs = []
    ctx.consume(rec)
    m = diff_tables(ctx.read_tables(), want, S, W)
    if m:
        msgs.append("trace fold: " + m)
    ctx.reset()
    ik.trace_fold(ctx, blocks_per_segment=int(rng.integers(0, 5)), serial=bool(rng.integers(0, 2)))
    m = diff_tables(ctx.read_tables(), want, S, W)
    if m:
        msgs.append("online: " + m)
    ctx.reset()
    ik.run(mask | smem, ctx)
    t = ctx.read_tables()
    w2 = want.copy()
    w2[0:4] = 0
    m = diff_tables(t, w2, S, W)
    if m:
        msgs.append("inline: " + m)
    ctx.close()
    ik.close()
    if msgs:
        fails += 1
        print("FAIL case %d %s size %d mask %d smem %d seed %d: %s" % (case, name, size, mask, smem, seed,
                                                                      "; ".join(msgs)), flush=True)
torch.cuda.synchronize()
print("fuzz inline: %d cases, %d failures" % (n_cases, fails))
sys.exit(1 if fails else 0)
