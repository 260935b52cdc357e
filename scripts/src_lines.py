"""Per-CUDA-line totals (warp-instructions executed, stall samples) of one kernel in an
ncu report, from `ncu -i REP --page source --print-source cuda,sass --csv`.
Usage: python scripts/src_lines.py REP KERNEL_REGEX [top]"""
import collections
import csv
import io
import subprocess
import sys

rep, kern = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
txt = subprocess.run(["ncu", "-i", rep, "-k", f"regex:{kern}", "--page", "source", "--print-source", "cuda,sass",
                      "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
fname, cur, hdr = "?", None, None
exe = collections.Counter()
smp = collections.Counter()
src = {}
seen_fn = 0
for r in rows:
    if not r:
        continue
    if r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if r[0] == "Function Name":
        seen_fn += 1
        continue
    if r[0] == "Line No":
        hdr = r
        ie, isamp = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
        continue
    if seen_fn > 1:
        break
    if hdr is None:
        continue
    if r[0]:
        cur = (fname, int(r[0]))
        src[cur] = r[1]
    elif cur:
        try:
            exe[cur] += int(float(r[ie] or 0))
            smp[cur] += int(float(r[isamp] or 0))
        except ValueError:
            pass
te, ts = sum(exe.values()), sum(smp.values())
print(f"{kern}: {te:,} warp-instr, {ts} samples")
for k in sorted(exe, key=lambda k: -exe[k])[:top]:
    print(f"{k[0][:14]:14s}:{k[1]:4d} {exe[k] / te * 100:5.1f}% {smp[k] / max(ts, 1) * 100:5.1f}%  {src[k].strip()[:90]}")
