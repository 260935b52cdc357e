"""Summarise gpurun_out/raw_f{0,1,2}.csv (ncu --set full, one launch per kernel per NYX field) into
profiles/<round>_ncu_full_summary.json: {field: {kernel: {time_us, dram_bytes, dram_read, dram_write,
inst_executed, issue_active_pct, alu_pct, fma_pct, lsu_pct, warps_active_pct, regs, grid, block}}}
and the launch list (gpurun_out/launches_bench.csv) into <round>_launches_share.txt.
Usage: python scripts/ncu_fields_summary.py r02"""
import csv
import json
import os
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
G, P = os.path.join(ROOT, "gpurun_out"), os.path.join(ROOT, "profiles")
rnd = sys.argv[1] if len(sys.argv) > 1 else "r02"
names = {0: "density", 1: "velocity", 2: "temperature"}
want = {
    "time_us": ("gpu__time_duration.sum", 1e-3),
    "dram_read": ("dram__bytes_read.sum", 1),
    "dram_write": ("dram__bytes_write.sum", 1),
    "inst_executed": ("smsp__inst_executed.sum", 1),
    "issue_active_pct": ("sm__inst_issued.avg.pct_of_peak_sustained_active", 1),
    "alu_pct": ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", 1),
    "fma_pct": ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", 1),
    "lsu_pct": ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", 1),
    "warps_active_pct": ("sm__warps_active.avg.pct_of_peak_sustained_active", 1),
    "regs": ("launch__registers_per_thread", 1),
    "grid": ("launch__grid_size", 1),
    "block": ("launch__block_size", 1),
}
unit_scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9, "B": 1,
              "nsecond": 1, "usecond": 1e3, "msecond": 1e6, "ns": 1, "us": 1e3, "ms": 1e6}
out = {}
for f, fname in names.items():
    path = os.path.join(G, f"raw_f{f}.csv")
    if not os.path.exists(path):
        continue
    rows = list(csv.reader(open(path)))
    hdr, units = rows[0], rows[1]
    col = {h: i for i, h in enumerate(hdr)}
    res = {}
    for r in rows[2:]:
        k = r[col["Kernel Name"]].split("(")[0].replace("void ", "").strip()
        d = {}
        for key, (m, sc) in want.items():
            if m not in col:
                continue
            v = r[col[m]].replace(",", "")
            try:
                x = float(v)
            except ValueError:
                continue
            u = units[col[m]]
            if key == "time_us":
                x = x * unit_scale.get(u, 1) / 1e3
            elif key.startswith("dram"):
                x = x * unit_scale.get(u, 1)
            d[key] = x
        if "dram_read" in d and "dram_write" in d:
            d["dram_bytes"] = d["dram_read"] + d["dram_write"]
        res[k] = d
    out[fname] = res
json.dump(out, open(os.path.join(P, f"{rnd}_ncu_full_summary.json"), "w"), indent=1)
lp = os.path.join(G, "launches_bench.csv")
if os.path.exists(lp):
    rows = [r for r in csv.reader(open(lp)) if r]
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    ik, im, iv = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    tot, cnt = defaultdict(float), defaultdict(int)
    for r in rows[hi + 1:]:
        if len(r) <= iv or r[im] != "gpu__time_duration.sum":
            continue
        nm = r[ik].split("(")[0].replace("void ", "").strip()
        if "szx::" not in nm and not nm.startswith("k_"):
            continue
        tot[nm] += float(r[iv].replace(",", ""))
        cnt[nm] += 1
    allt = sum(tot.values()) or 1
    with open(os.path.join(P, f"{rnd}_launches_share.txt"), "w") as fo:
        fo.write("# ncu --metrics gpu__time_duration.sum --clock-control none, python bench.py --steps 3 --warmup 1 "
                 "--no-graph (3 NYX fields per step)\n# kernel / launches / mean ns / share of library kernel time "
                 "(cold-cache, serialised)\n")
        for k in sorted(tot, key=lambda k: -tot[k]):
            fo.write(f"{k:60s} launches={cnt[k]:3d} mean_ns={tot[k] / cnt[k]:10.0f} share={tot[k] / allt * 100:5.1f}%\n")
    os.replace(lp, os.path.join(P, f"{rnd}_launches_bench.csv"))
print(json.dumps({f: {k: {kk: round(vv, 1) for kk, vv in v.items() if kk in ("time_us", "dram_bytes", "issue_active_pct")}
                      for k, v in d.items()} for f, d in out.items()}, indent=0)[:3000])
