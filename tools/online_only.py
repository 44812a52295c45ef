"""bench.py's online-trace measurement alone (all four kernels), printed per kernel."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import bench  # noqa: E402

out = bench.measure_online_trace(torch.device("cuda", 0))
for k, v in out.items():
    print(k, json.dumps({x: v[x] for x in ("online_ms", "serial_ms", "K_online", "records", "segments")}))
