"""Per-(file, line) totals of warp-instructions and stall samples of one kernel, over every
source file of `ncu -i REP -k regex:K --page source --print-source cuda,sass --csv`.
Usage: python scripts/src_lines_all.py CSV units [top]  (units: divide instruction counts)"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
units = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
fname, hdr, line, src = "?", None, None, {}
ins, smp = collections.Counter(), collections.Counter()
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] in ("Function Name",):
        continue
    if r[0] == "Line No":
        hdr = r
        ie, ist = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
        continue
    if hdr is None:
        continue
    if r[0]:
        line = (fname, int(r[0]))
        src[line] = r[1]
        continue
    try:
        ins[line] += int(r[ie])
        smp[line] += int(r[ist])
    except (ValueError, IndexError):
        pass
ti, ts = sum(ins.values()), sum(smp.values())
print(f"total {ti / units:.1f} warp-inst per unit, {ts} samples")
for l, n in ins.most_common(top):
    print(f"{l[0][:14]:14s}:{l[1]:5d} {n / units:7.2f} {100 * smp[l] / max(ts, 1):5.1f}%  {src.get(l, '')[:80]}")
