"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list into profiles/ markdown.
usage: python tools/launch_list.py launches.csv out.md ["bench command line"]"""
import collections
import csv
import sys

SCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
STEP = ("consume_kernel", "init_tables_kernel", "block_sums_kernel", "scan_bsums_kernel",
        "scan_apply_kernel", "draw_kernel", "pack_kernel", "unpack_kernel")
rows = list(csv.reader(open(sys.argv[1])))
hdr, data = None, []
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        data.append(dict(zip(hdr, r)))
agg = collections.defaultdict(lambda: [0, 0.0])
for d in data:
    name = d["Kernel Name"].split("(")[0].replace("void ", "")
    agg[name][0] += 1
    agg[name][1] += float(d["Metric Value"].replace(",", "")) * SCALE[d["Metric Unit"]]
tot = sum(v[1] for v in agg.values())
step = {k: v for k, v in agg.items() if any(s in k for s in STEP)}
stot = sum(v[1] for v in step.values())
cmd = sys.argv[3] if len(sys.argv) > 3 else (
    "python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu-baseline --no-slowdown --no-injection")
out = ["# Launch list: `%s`" % sys.argv[1].split("/")[-1], "",
       "ncu --metrics gpu__time_duration.sum --clock-control none over `%s` (generation included). "
       "Per-launch times are cold-cache and serialised: compare shares, not absolutes." % cmd, "",
       "## Kernels of the timed step (reset + consume + sampling)", "",
       "| kernel | launches | total ms | share of step |", "|---|---|---|---|"]
for k, (n, t) in sorted(step.items(), key=lambda x: -x[1][1]):
    out.append("| `%s` | %d | %.3f | %.1f %% |" % (k[:70], n, t, 100 * t / stot))
out += ["", "## Everything in the process", "", "| kernel | launches | total ms | share |", "|---|---|---|---|"]
for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
    out.append("| `%s` | %d | %.3f | %.1f %% |" % (k[:70], n, t, 100 * t / tot))
open(sys.argv[2], "w").write("\n".join(out) + "\n")
print("\n".join(out[:14]))
