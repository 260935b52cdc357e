"""Summarise an ncu --page source --print-source sass CSV: top instructions by executed count
and stall samples, plus opcode histogram weighted by execution count."""
import csv
import collections
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
ia, isrc, iexe, isamp = hdr.index("Address"), hdr.index("Source"), hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
data = []
for r in rows[2:]:
    try:
        data.append((r[ia], r[isrc], int(float(r[iexe] or 0)), int(float(r[isamp] or 0))))
    except (ValueError, IndexError):
        pass
tot = sum(d[2] for d in data)
samp = sum(d[3] for d in data)
print(f"{len(data)} SASS instrs, executed {tot:,} warp-instr, {samp} stall samples")
op = collections.Counter()
for a, s, e, _ in data:
    op[s.split()[0] if not s.startswith("@") else s.split()[1]] += e
print("opcodes:", ", ".join(f"{k}:{v/tot*100:.1f}%" for k, v in op.most_common(25)))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 30
print("--- top by stall samples")
for a, s, e, sm in sorted(data, key=lambda d: -d[3])[:n]:
    print(f"{a} {sm:6d} {e:10d}  {s[:90]}")
