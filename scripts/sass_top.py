"""Summarise an ncu --page source --print-source sass CSV (first kernel instance):
opcode histogram weighted by executions, and the hottest instructions."""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
# first section: row 0 = kernel name, row 1 = header, rows until next "Kernel Name"
hdr = rows[1]
data = []
for r in rows[2:]:
    if r and r[0] == "Kernel Name":
        break
    data.append(r)
ia, isrc = hdr.index("Address"), hdr.index("Source")
iexe, isamp = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
D = []
for r in data:
    try:
        D.append((r[ia][-5:], r[isrc], int(float(r[iexe] or 0)), int(float(r[isamp] or 0))))
    except (ValueError, IndexError):
        pass
tot = sum(d[2] for d in D)
print(f"{len(D)} SASS instrs, executed {tot:,} warp-instr, {sum(d[3] for d in D)} stall samples")
op = collections.Counter()
for a, s, e, _ in D:
    t = s.split()
    op[t[1] if t and t[0].startswith("@") else (t[0] if t else "?")] += e
print("opcodes:", ", ".join(f"{k}:{v / tot * 100:.1f}%" for k, v in op.most_common(22)))
thr = int(sys.argv[2]) if len(sys.argv) > 2 else 0
if thr:
    for a, s, e, sm in D:
        if e >= thr:
            print(f"{a} {e:9d} {sm:5d}  {s[:80]}")
