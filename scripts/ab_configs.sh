#!/bin/bash
# A/B of experiment builds (build_exp/*.so via SZX_LIB) on the small configurations
# (CESM / Hurricane, L2 flushed, CUDA graphs): compress / decompress us and fractions.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for f in ${VARIANTS:-build_exp/*.so}; do
  SZX_LIB=$PWD/$f timeout 600 python scripts/bench_configs.py --only ${ONLY:-cesm,hurricane} --iters ${ITERS:-20} \
      > gpurun_out/abc.jsonl 2>gpurun_out/abc.err || tail -3 gpurun_out/abc.err
  python3 - "$f" <<'PY'
import json, sys
print(sys.argv[1])
for l in open("gpurun_out/abc.jsonl"):
    d = json.loads(l)
    print("  %-10s nc=%.3f c=%6.1f d=%6.1f us  cf=%.3f df=%.3f " % (d["config"], d["nonconst_frac"], d["compress_ms"] * 1e3,
          d["decompress_ms"] * 1e3, d["compress_hbm_frac"], d["decompress_hbm_frac"]),
          {k: round(v * 1e3, 1) for k, v in d["kernels_ms"].items()})
PY
done
