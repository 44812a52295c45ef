"""One online trace fold (default segments) of an instrumented kernel, for ncu:
python tools/prof_online.py KERNEL [SIZE]"""
import sys

import torch

sys.path.insert(0, ".")
from paper_conf_isca_stephensonhlejn15_b200 import sassi  # noqa: E402

ik = sassi.InstrumentedKernel(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 0)
ctx = ik.context(sassi.SASSI_H_EVERY)
print(ik.trace_fold(ctx))
torch.cuda.synchronize()
