#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_lm.py -m gpu -x -q -k "race or never_blocks or fork_explores or graph_replay" > gpurun_out/r3z_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3z_pytest.log
for r in 1 2; do
  ASTRA_DUMP_REPORT=gpurun_out/r3z_report_$r.json python bench.py --no-cpu-baseline >> gpurun_out/r3z_bench.log 2>&1
done
python bench.py --batch 64 --no-cpu-baseline > gpurun_out/r3z_bench_b64.log 2>&1
