#!/bin/bash
# compress + decompress kernel times of each experiment build in build_exp/ (FIELDS, default velocity, density)
cd "$(dirname "$0")/.."
for F in ${FIELDS:-1 0}; do
  for f in build_exp/*.so; do
    SZX_LIB=$PWD/$f FIELD=$F STEPS=${STEPS:-30} timeout 300 python scripts/time_codec.py 2>&1 | tail -1
  done
done
