#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "small_batch_persistent_forward" > gpurun_out/r2_t37.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t37.log
V64="a1=256.1.1.2,rec=64.1.1,bptt=128.1.1,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=128.1.1,hdy=128.1.1,wg_side=1,fwd=3,bwd=0,pf=2,hov=0,gc=3,wgs=1,bpw=1"
for i in 1 2; do ASTRA_VARIANT="$V64" timeout 300 python bench.py --profile --steps 10 --batch 64 >> gpurun_out/r2_prof37.log 2>&1; done
