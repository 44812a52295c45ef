"""Run one instrumented kernel in one mode a few times (for ncu): python tools/prof_ik.py NAME MODE [REPS]"""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_isca_stephensonhlejn15_b200 import sassi  # noqa: E402

name, mode = sys.argv[1], int(sys.argv[2])
reps = int(sys.argv[3]) if len(sys.argv) > 3 else 2
ik = sassi.InstrumentedKernel(name, 0)
ctx = ik.context(sassi.SASSI_H_EVERY)
for _ in range(reps):
    ik.run(mode, ctx if mode & sassi.SASSI_H_EVERY else None)
torch.cuda.synchronize()
