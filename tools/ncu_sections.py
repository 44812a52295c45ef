"""Instructions executed / stall samples per code section (line ranges) from a cuda,sass csv.
usage: ncu_sections.py CSV FILE name:start-end ..."""
import csv
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
target = sys.argv[2]
secs = []
for a in sys.argv[3:]:
    n, r = a.split(":")
    lo, hi = r.split("-")
    secs.append((n, int(lo), int(hi)))
fname = ""
agg = defaultdict(lambda: [0, 0])
tot = tst = 0
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] not in ("", "Line No", "Function Name") and len(r) > 8:
        try:
            ln, e, s = int(r[0]), int(r[7] or 0), int(r[4] or 0)
        except ValueError:
            continue
        tot += e
        tst += s
        k = "other:" + fname
        if fname == target:
            for n, lo, hi in secs:
                if lo <= ln <= hi:
                    k = n
                    break
        agg[k][0] += e
        agg[k][1] += s
for k, (e, s) in sorted(agg.items(), key=lambda x: -x[1][0]):
    print("%-32s exec %5.1f%%  stall %5.1f%%  (%d)" % (k, 100 * e / tot, 100 * s / max(tst, 1), e))
