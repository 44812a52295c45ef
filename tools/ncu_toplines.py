"""Top source lines of one file by instructions executed / stall samples, from an ncu report:
python tools/ncu_toplines.py REPORT.ncu-rep consume.cu [N]"""
import csv
import subprocess
import sys
from collections import defaultdict

rep, target = sys.argv[1], sys.argv[2]
N = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
ex, st, src = defaultdict(int), defaultdict(int), {}
fname, hdr = "", None
tot_e = tot_s = 0
for r in csv.reader(out.splitlines()):
    if len(r) == 2 and r[0] in ("File Path", "File Name"):
        fname = r[1].split("/")[-1]
        continue
    if r and r[0] == "Line No":
        hdr = {k: i for i, k in enumerate(r)}
        continue
    if hdr and r and len(r) > 8:
        try:
            if not r[0]:
                continue
            line = int(r[0])
            e = int(r[hdr["Instructions Executed"]] or 0)
            s = int(r[hdr["Warp Stall Sampling (All Samples)"]] or 0)
        except (ValueError, KeyError):
            continue
        key = (fname, line)
        ex[key] += e
        st[key] += s
        src[key] = r[1]
        tot_e += e
        tot_s += s
print("total instructions %.4e  stall samples %d" % (tot_e, tot_s))
for k in sorted(ex, key=lambda k: -ex[k])[:N]:
    print("%-14s %4d %6.2f%% %6.2f%%  %s" % (k[0][:14], k[1], 100 * ex[k] / tot_e, 100 * st[k] / max(tot_s, 1),
                                         src[k].strip()[:90]))
