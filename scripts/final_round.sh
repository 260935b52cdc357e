#!/bin/bash
# End-of-round evidence on one GPU: smoke, the GPU test suite, the bench line, per-field ncu --set full
# summaries + the bench launch list, and the per-config sweep (all outputs under gpurun_out/).
cd "$(dirname "$0")/.."
mkdir -p gpurun_out
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err; echo "bench rc=$?"
bash scripts/ncu_fields.sh
timeout 900 python scripts/bench_configs.py --iters 20 > gpurun_out/configs_final.jsonl 2> gpurun_out/configs_final.err; echo "configs rc=$?"
tail -2 gpurun_out/smoke.log; tail -3 gpurun_out/pytest_gpu.log
