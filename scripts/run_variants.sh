#!/bin/bash
# time bench.py with each experiment build in build_exp/ (kernel ms per launch)
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
for f in build_exp/*.so; do
  SZX_LIB=$PWD/$f timeout 300 python bench.py --steps ${STEPS:-100} --warmup 5 --no-cpu --no-e2e ${BENCH_ARGS} > gpurun_out/v.json 2>gpurun_out/v.err
  python3 -c "
import json,sys; d=json.loads(open('gpurun_out/v.json').readline())
print('$f', {k:round(v*1000,1) for k,v in d['kernels_ms_per_launch'].items()}, round(d['ms_per_step']*1000,1))" || tail -3 gpurun_out/v.err
done
