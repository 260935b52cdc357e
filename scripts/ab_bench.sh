#!/bin/bash
# A/B of experiment builds (build_exp/*.so, loaded via SZX_LIB) on the bench workload:
# per field compress / decompress ms and per-kernel ms per launch.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for f in ${VARIANTS:-build_exp/*.so}; do
  SZX_LIB=$PWD/$f timeout 600 python bench.py --steps ${STEPS:-30} --warmup 5 --no-cpu --no-e2e ${BENCH_ARGS} > gpurun_out/v.json 2>gpurun_out/v.err
  python3 - "$f" <<'PY' || tail -5 gpurun_out/v.err
import json, sys
d = json.loads(open("gpurun_out/v.json").readline())
print(sys.argv[1], "step_ms=%.1f" % (d["ms_per_step"] * 1000 / 1000), "graph=%s" % d.get("graph"))
for k, r in d["fields"].items():
    print("  %-12s c=%6.1f d=%6.1f us  cf=%.3f df=%.3f  " % (k, r["compress_ms"] * 1e3, r["decompress_ms"] * 1e3,
          r["compress_hbm_frac"], r["decompress_hbm_frac"]),
          {kk: round(v * 1e3, 1) for kk, v in r["kernels_ms_per_launch"].items()})
PY
done
