"""Turn gpurun_out/ (ncu launch list + --set full report + bench line) into
profiles/<round>_*.  Usage: python scripts/summarize_profiles.py r01"""
import csv
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
rnd = sys.argv[1] if len(sys.argv) > 1 else "r01"
G = os.path.join(ROOT, "gpurun_out")
P = os.path.join(ROOT, "profiles")
os.makedirs(P, exist_ok=True)

# 1) launch list (per-launch device time, cold-cache, serialised): shares per kernel
rows = [r for r in csv.reader(open(os.path.join(G, "launches_bench.csv"))) if r]
hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
hdr = rows[hdr_i]
ik, im, iv = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
tot = defaultdict(float)
cnt = defaultdict(int)
for r in rows[hdr_i + 1:]:
    if len(r) <= iv or r[im] != "gpu__time_duration.sum":
        continue
    name = r[ik].split("(")[0].replace("void ", "").strip()
    if not name.startswith("szx::"):
        continue
    tot[name] += float(r[iv].replace(",", ""))
    cnt[name] += 1
allt = sum(tot.values())
with open(os.path.join(P, f"{rnd}_launches_share.txt"), "w") as f:
    f.write("# ncu --metrics gpu__time_duration.sum --clock-control none, python bench.py --steps 3 --warmup 1\n")
    f.write("# per-kernel total / launches / mean (ns) / share of library kernel time (cold-cache, serialised)\n")
    for k in sorted(tot, key=lambda k: -tot[k]):
        f.write(f"{k:45s} launches={cnt[k]:3d} mean_ns={tot[k] / cnt[k]:10.0f} share={tot[k] / allt * 100:5.1f}%\n")
os.replace(os.path.join(G, "launches_bench.csv"), os.path.join(P, f"{rnd}_launches_bench.csv"))

# 2) --set full capture: per-kernel counters (one warm launch each)
raw = subprocess.run(["ncu", "-i", os.path.join(G, "prof_full.ncu-rep"), "--page", "raw", "--csv"],
                     capture_output=True, text=True).stdout
rr = list(csv.reader(raw.splitlines()))
h = rr[0]
want = {"time_ns": "gpu__time_duration.sum", "dram_read": "dram__bytes_read.sum",
        "dram_write": "dram__bytes_write.sum",
        "dram_pct_peak": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "issue_active_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "alu_pct": "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "lsu_pct": "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "warps_active_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
        "inst_executed_warp": "smsp__inst_executed.sum", "registers": "launch__registers_per_thread",
        "grid": "launch__grid_size", "block": "launch__block_size"}
units = rr[1]
out = {}
for r in rr[2:]:
    name = r[h.index("Kernel Name")].split("(")[0].replace("void ", "").strip()
    d = {}
    for k, m in want.items():
        if m in h:
            v = r[h.index(m)].replace(",", "")
            u = units[h.index(m)]
            try:
                x = float(v)
                if u == "Mbyte":
                    x *= 1e6
                elif u == "Kbyte":
                    x *= 1e3
                elif u == "Gbyte":
                    x *= 1e9
                elif u in ("usecond", "us"):
                    x *= 1e3
                elif u in ("msecond", "ms"):
                    x *= 1e6
                d[k] = x
            except ValueError:
                d[k] = v
    d["dram_bytes"] = d.get("dram_read", 0) + d.get("dram_write", 0)
    out.setdefault(name, d)
json.dump(out, open(os.path.join(P, f"{rnd}_ncu_full_summary.json"), "w"), indent=1)
with open(os.path.join(P, f"{rnd}_ncu_full_summary.txt"), "w") as f:
    f.write("# ncu --set full --clock-control none, scripts/prof_nyx.py (NYX 512^3 f32 REL 1e-3), one warm launch each\n")
    for k, d in out.items():
        f.write(f"{k}\n  " + " ".join(f"{a}={b:.4g}" if isinstance(b, float) else f"{a}={b}" for a, b in d.items()) + "\n")
# 3) bench line
if os.path.exists(os.path.join(G, "bench.json")):
    os.replace(os.path.join(G, "bench.json"), os.path.join(P, f"{rnd}_bench.json"))
print(open(os.path.join(P, f"{rnd}_launches_share.txt")).read())
print(open(os.path.join(P, f"{rnd}_ncu_full_summary.txt")).read())
