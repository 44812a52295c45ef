"""Minimal synccheck reproduction: random edge traces through the memdiv fold (compute-sanitizer)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np  # noqa: E402

import oracle  # noqa: E402
from gpu_helpers import to_device, gpu_table  # noqa: E402
from test_oracle import random_trace  # noqa: E402

mask = int(sys.argv[1]) if len(sys.argv) > 1 else 2
s2, W, h2, a2, v2 = random_trace(4321, n=3000)
t = gpu_table(s2, W, mask, to_device(s2, h2, a2, v2))
assert np.array_equal(t, oracle.run(s2, W, mask, h2, a2, v2))
print("ok", mask)
