"""Stall reasons per CUDA source line of one kernel in an ncu report.
Usage: python scripts/stall_lines.py REP KERNEL_REGEX [top]"""
import collections
import csv
import io
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
txt = subprocess.run(["ncu", "-i", rep, "-k", f"regex:{kern}", "--page", "source", "--print-source", "cuda,sass",
                      "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr, cur, fn = None, None, 0
agg = collections.defaultdict(collections.Counter)
src = {}
for r in rows:
    if not r:
        continue
    if r[0] == "Function Name":
        fn += 1
        continue
    if r[0] == "Line No":
        hdr = r
        continue
    if r[0] == "File Path" or hdr is None or fn > 1:
        continue
    if r[0]:
        cur = int(r[0])
        src[cur] = r[1]
        continue
    for i, h in enumerate(hdr):
        if h.startswith("stall_") and "Not Issued" not in h:
            try:
                agg[cur][h[6:]] += int(float(r[i] or 0))
            except ValueError:
                pass
tot = collections.Counter()
for v in agg.values():
    tot.update(v)
T = sum(tot.values()) or 1
print("all:", {k: round(v / T * 100, 1) for k, v in tot.most_common(10)})
for ln in sorted(agg, key=lambda x: -sum(agg[x].values()))[:top]:
    print(ln, round(sum(agg[ln].values()) / T * 100, 1), agg[ln].most_common(3), src[ln].strip()[:70])
