"""Hot SASS of one kernel from its SASS page CSV: instructions in address order with
executed counts per unit, only those above a threshold.
Usage: python scripts/sass_hot.py CSV n_units [min_per_unit]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
units = float(sys.argv[2])
thr = float(sys.argv[3]) if len(sys.argv) > 3 else 0.2
hdr = rows[1]
ie, isrc = hdr.index("Instructions Executed"), hdr.index("Source")
ia = hdr.index("Address")
ist = hdr.index("Warp Stall Sampling (All Samples)")
for r in rows[2:]:
    if len(r) <= ie:
        continue
    try:
        n = int(r[ie])
    except ValueError:
        continue
    if n / units >= thr:
        print(f"{r[ia][-5:]} {n / units:6.2f} {r[ist]:>6s}  {r[isrc].strip()[:100]}")
