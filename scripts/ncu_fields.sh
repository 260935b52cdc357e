#!/bin/bash
# ncu --set full of every kernel of one compress + decompress step, per NYX field (one warm launch
# each), plus the ncu launch list of the bench command; summarised by scripts/ncu_fields_summary.py
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for F in 0 1 2; do
  FIELD=$F STEPS=2 timeout 900 ncu --set full --clock-control none --import-source on \
     -k "regex:k_block_stats|k_classify|k_encode|k_decode_w" -s 4 -c 4 \
     -o gpurun_out/prof_f$F -f python scripts/prof_nyx.py > gpurun_out/ncu_f$F.log 2>&1
  echo "field $F ncu rc=$?"
  ncu -i gpurun_out/prof_f$F.ncu-rep --page raw --csv > gpurun_out/raw_f$F.csv 2>/dev/null
  ncu -i gpurun_out/prof_f$F.ncu-rep --page details --csv > gpurun_out/det_f$F.csv 2>/dev/null
  rm -f gpurun_out/prof_f$F.ncu-rep
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
   --log-file gpurun_out/launches_bench.csv python bench.py --steps 3 --warmup 1 --no-cpu --no-e2e --no-kernels --no-graph \
   > gpurun_out/ncu_launch_bench.log 2>&1; echo "ncu launches rc=$?"
