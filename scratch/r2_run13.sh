#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_gemm.py -q -x > gpurun_out/r2_t13.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t13.log
V512="a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0"
for v in "rec=256.1.1.2" "rec=224.1.1.2" "rec=256.1.1" "rec=224.1.1.2,a1=224.1.1.2" "rec=256.1.1.2" "rec=224.1.1.2"; do
  ASTRA_VARIANT="$V512,$v" timeout 300 python bench.py --profile --steps 5 >> gpurun_out/r2_prof13.log 2>&1
done
