"""Opcode mix (warp-instructions executed, weighted) of one kernel's SASS page CSV
(`ncu -i REP -k regex:K --page source --print-source sass --csv`).
Usage: python scripts/sass_mix.py CSV [n_units]   (n_units: divide counts, e.g. blocks)"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
units = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
hdr = rows[1]
ie, isrc = hdr.index("Instructions Executed"), hdr.index("Source")
mix = collections.Counter()
tot = 0
for r in rows[2:]:
    if len(r) <= ie:
        continue
    try:
        n = int(r[ie])
    except ValueError:
        continue
    op = r[isrc].strip().split()
    if not op:
        continue
    o = op[0]
    if o.startswith("@"):
        o = op[1]
    o = o.split(".")[0]
    mix[o] += n
    tot += n
print(f"total {tot:,} warp-inst, {tot / units:.1f} per unit")
for o, n in mix.most_common(40):
    print(f"{o:10s} {n / units:8.2f} {n / tot * 100:5.1f}%")
