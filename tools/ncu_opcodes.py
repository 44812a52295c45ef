"""Per-opcode and per-(line, opcode) instruction counts from `ncu --page source --csv
--print-source cuda,sass` output: python tools/ncu_opcodes.py SRC.csv [N] [OPCODE_REGEX]"""
import csv
import re
import sys
from collections import Counter

rows = list(csv.reader(open(sys.argv[1])))
N = int(sys.argv[2]) if len(sys.argv) > 2 else 30
pat = re.compile(sys.argv[3]) if len(sys.argv) > 3 else None
hdr, cur, fname = None, None, ""
ops, lines, tot = Counter(), Counter(), 0
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = 1
        continue
    if not hdr or len(r) < 8:
        continue
    if r[0]:
        cur = (fname, int(r[0]), r[1].strip()[:70])
        continue
    toks = [t for t in r[3].split() if not t.startswith("@")]
    if not toks:
        continue
    try:
        e = int(r[7] or 0)
    except ValueError:
        continue
    op = toks[0]
    ops[op] += e
    tot += e
    if pat is None or pat.search(op):
        lines[(cur, op)] += e
print("total %.4e" % tot)
for k, v in ops.most_common(N):
    print("%-30s %6.2f%%" % (k, 100 * v / tot))
print()
for (c, op), v in lines.most_common(N):
    print("%6.2f%% %-22s %s" % (100 * v / tot, op, c))
