#!/bin/bash
mkdir -p gpurun_out
for w in 400 0 400; do
  ASTRA_DUMP_REPORT=gpurun_out/r3tw_report_$w.json python bench.py --no-cpu-baseline --tune-warmup $w >> gpurun_out/r3tw_bench.log 2>&1
done
