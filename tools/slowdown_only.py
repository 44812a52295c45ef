import json, sys, torch
sys.path.insert(0, ".")
import bench
print(json.dumps(bench.measure_slowdown(torch.device("cuda:0"))))
