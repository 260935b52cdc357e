#!/bin/bash
# Source-level ncu capture of the encode/decode kernels on an all-nonconstant field
# (NYX velocity-like, FIELD=1): one warm launch each, then per-SASS CSVs for reading here.
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
K=${KERNELS:-"k_enc_size|k_enc_write|k_decode_w|k_encode"}
FIELD=${FIELD:-1} timeout 1200 ncu --set full --clock-control none --import-source on -k "regex:${K}" \
    -s ${SKIP:-4} -c ${COUNT:-3} -o gpurun_out/prof_src -f python scripts/prof_nyx.py > gpurun_out/ncu_src.log 2>&1
echo "ncu rc=$?"; tail -2 gpurun_out/ncu_src.log
for k in $(echo $K | tr '|' ' '); do
  ncu -i gpurun_out/prof_src.ncu-rep -k "regex:$k" --page source --print-source sass --csv > gpurun_out/src_$k.csv 2>/dev/null
  ncu -i gpurun_out/prof_src.ncu-rep -k "regex:$k" --page details --csv > gpurun_out/det_$k.csv 2>/dev/null
done
ls -la gpurun_out/src_*.csv
