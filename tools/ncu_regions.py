"""Aggregate per-source-line instruction counts / stall samples of one file into named line
ranges: python tools/ncu_regions.py SRC.csv consume.cu name:lo-hi[,lo-hi] ...
(the csv is `ncu -i X --page source --csv --print-source cuda,sass`; lines of other files
(intrinsic headers) are attributed to 'intrinsics')."""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
target = sys.argv[2]
regions = []
for spec in sys.argv[3:]:
    name, rng = spec.split(":")
    for part in rng.split(","):
        lo, hi = part.split("-")
        regions.append((name, int(lo), int(hi)))
ex, st = defaultdict(int), defaultdict(int)
fname, hdr = "", None
tot_e = tot_s = 0
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr and r and r[0] not in ("", "Function Name") and len(r) > 8:
        try:
            line, e, s = int(r[0]), int(r[7] or 0), int(r[4] or 0)
        except ValueError:
            continue
        name = "intrinsics" if fname != target else "other"
        if fname == target:
            for n, lo, hi in regions:
                if lo <= line <= hi:
                    name = n
                    break
        ex[name] += e
        st[name] += s
        tot_e += e
        tot_s += s
nb = float(sys.argv[0] and 1)
print("total instructions %.3e, stall samples %d" % (tot_e, tot_s))
for n in sorted(ex, key=lambda k: -ex[k]):
    print("%-12s %6.2f%% instr  %6.2f%% stall  %.3e" % (n, 100 * ex[n] / tot_e, 100 * st[n] / max(tot_s, 1), ex[n]))
