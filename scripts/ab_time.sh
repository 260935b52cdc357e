#!/bin/bash
# kernel times of each build_exp/*.so on the given NYX fields (no parity check)
cd "$(dirname "$0")/.."
for F in ${FIELDS:-0 1}; do echo "field $F"; BENCH_ARGS="--field $F" STEPS=${STEPS:-50} bash scripts/run_variants.sh; done
