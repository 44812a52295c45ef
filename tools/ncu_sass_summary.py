"""Summarise an ncu source-page SASS csv: instruction mix and stall samples by opcode / address."""
import csv
import re
import sys
from collections import defaultdict

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
idx = {h: i for i, h in enumerate(hdr)}
data = rows[2:]
ex = defaultdict(int)
st = defaultdict(int)
tot_ex = tot_st = 0
per = []
for r in data:
    if len(r) < len(hdr):
        continue
    src = r[idx["Source"]]
    op = src.split()[0] if src else "?"
    if op.startswith("@"):
        op = src.split()[1]
    op = re.sub(r"\..*", "", op)
    e = int(r[idx["Instructions Executed"]] or 0)
    s = int(r[idx["Warp Stall Sampling (All Samples)"]] or 0)
    ex[op] += e
    st[op] += s
    tot_ex += e
    tot_st += s
    per.append((s, e, r[idx["Address"]], src))
print("total executed %d, stall samples %d" % (tot_ex, tot_st))
print("%-10s %8s %8s" % ("opcode", "exec%", "stall%"))
for op in sorted(ex, key=lambda o: -ex[o])[:30]:
    print("%-10s %7.2f%% %7.2f%%" % (op, 100 * ex[op] / tot_ex, 100 * st[op] / max(tot_st, 1)))
print("\ntop stall instructions:")
stall_cols = [h for h in hdr if h.startswith("stall_")]
for s, e, a, src in sorted(per, reverse=True)[:25]:
    print("%6.2f%% %10d %s %s" % (100 * s / max(tot_st, 1), e, a, src[:70]))
