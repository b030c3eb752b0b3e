#!/bin/bash
mkdir -p gpurun_out/r2_sanitize2
for c in rec_persist rhn_fused bptt_persist scrn_persist gemm_kb rec_fused bptt_fused; do
  for tool in memcheck racecheck synccheck; do
    timeout 900 compute-sanitizer --tool $tool  python scratch/sanitize_cases.py $c > gpurun_out/r2_sanitize2/${c}_${tool}.log 2>&1
    echo "rc=$?" >> gpurun_out/r2_sanitize2/${c}_${tool}.log
  done
done
