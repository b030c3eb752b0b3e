#!/bin/bash
mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_cell.py -q -x -k "persistent_bptt" > gpurun_out/r2_t17.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t17.log
V64="a1=256.1.1.2,rec=64.1.1,bptt=128.1.1,du=256.1.1.2,dw=224.1.1.2,dx=224.1.1.2,head=256.1.1,wg_side=1,fwd=3,pf=2,hov=0,gc=3,bpw=1"
for v in "bwd=0,wgs=1" "bwd=2" "bwd=0,wgs=1" "bwd=2"; do
  ASTRA_VARIANT="$V64,$v" timeout 300 python bench.py --profile --steps 10 --batch 64 >> gpurun_out/r2_prof17.log 2>&1
done
