#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py -q -x -k "wgrad_schedule or stream_schedules or graph_replay or gate_chunking" > gpurun_out/r2_t4.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t4.log
V512="a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0"
for w in 0 1 2; do
  ASTRA_VARIANT="$V512,wgs=$w" timeout 300 python bench.py --profile --steps 5 >> gpurun_out/r2_prof4.log 2>&1
done
V64="a1=256.1.1.2,rec=64.1.1,bptt=128.1.1,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=3,bwd=0,pf=2,hov=0"
for w in 0 1 2; do
  ASTRA_VARIANT="$V64,wgs=$w" timeout 300 python bench.py --profile --steps 5 --batch 64 >> gpurun_out/r2_prof4.log 2>&1
done
mkdir -p gpurun_out/sanitize
for c in rec_fused rec_persist bptt_fused rhn_fused; do
  for tool in memcheck racecheck synccheck; do
    timeout 600 compute-sanitizer --tool $tool --print-limit 20 python scratch/sanitize_cases.py $c > gpurun_out/sanitize/${c}_${tool}.log 2>&1
    echo "exit=$?" >> gpurun_out/sanitize/${c}_${tool}.log
  done
done
