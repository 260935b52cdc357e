#!/bin/bash
# A/B of encoder variants (build_exp/*.so): parity of each variant, then kernel times
# on the NYX density (field 0) and velocity (field 1) fields.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for f in build_exp/*.so; do
  SZX_LIB=$PWD/$f timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_dist.py -x -q 2>&1 | tail -1 | sed "s|^|$f: |"
done
for F in ${FIELDS:-0 1}; do echo "field $F"; BENCH_ARGS="--field $F" STEPS=50 bash scripts/run_variants.sh; done
