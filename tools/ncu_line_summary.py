"""Per-source-line instructions executed and stall samples from `ncu --page source --csv
--print-source cuda,sass` output."""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
out = []
fname = ""
hdr = None
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr and r and r[0] not in ("", "Function Name") and len(r) > 8:
        try:
            ex = int(r[7] or 0)
            st = int(r[4] or 0)
        except ValueError:
            continue
        out.append((ex, st, fname, r[0], r[1]))
tot = sum(o[0] for o in out)
tst = sum(o[1] for o in out)
print("total exec %d  stall %d" % (tot, tst))
for ex, st, f, ln, src in sorted(out, reverse=True)[: int(sys.argv[2]) if len(sys.argv) > 2 else 45]:
    print("%6.2f%% %6.2f%% %s:%s  %s" % (100 * ex / tot, 100 * st / max(tst, 1), f, ln, src.strip()[:80]))
