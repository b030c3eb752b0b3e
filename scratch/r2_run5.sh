#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py -q -x -k "bwd_pointwise_forms or fused_bwd or recompute" > gpurun_out/r2_t5.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t5.log
V512="a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0"
for f in 1 0 1 0; do
  ASTRA_VARIANT="$V512,bpw=$f" timeout 300 python bench.py --profile --steps 5 >> gpurun_out/r2_prof5.log 2>&1
done
V64="a1=256.1.1.2,rec=64.1.1,bptt=128.1.1,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=3,bwd=0,pf=2,hov=0"
for f in 1 0; do
  ASTRA_VARIANT="$V64,bpw=$f" timeout 300 python bench.py --profile --steps 5 --batch 64 >> gpurun_out/r2_prof5.log 2>&1
done
