#!/bin/bash
# ncu --set full of the main kernels (one launch each, after warm-up) + a launch list.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
K=${KERNELS:-"k_block_stats|k_classify|k_encode|k_index|k_decode"}
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
    --log-file gpurun_out/launches.csv python scripts/prof_nyx.py > gpurun_out/ncu_launch.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k "regex:${K}" -s ${SKIP:-5} -c ${COUNT:-5} \
    -o gpurun_out/prof_full -f python scripts/prof_nyx.py > gpurun_out/ncu_full.log 2>&1
echo "ncu rc=$?"; tail -3 gpurun_out/ncu_full.log
