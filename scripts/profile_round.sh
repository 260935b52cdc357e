#!/bin/bash
# Evidence for profiles/: bench line, ncu launch list of the bench command,
# ncu --set full of every kernel (one warm launch each), clocks.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw --format=csv > gpurun_out/gpu.txt 2>&1
lscpu > gpurun_out/lscpu.txt 2>&1
timeout 900 python bench.py ${BENCH_ARGS} > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/launches_bench.csv python bench.py --steps 3 --warmup 1 --no-cpu --no-e2e --no-fields \
   > gpurun_out/ncu_launch_bench.log 2>&1; echo "ncu launches rc=$?"
timeout 1500 ncu --set full --clock-control none --import-source on \
   -k "regex:k_block_stats|k_classify|k_enc_size|k_zscan|k_enc_write|k_decode" -s 6 -c 6 \
   -o gpurun_out/prof_full -f python scripts/prof_nyx.py > gpurun_out/ncu_full.log 2>&1; echo "ncu full rc=$?"
