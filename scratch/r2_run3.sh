#!/bin/bash
mkdir -p gpurun_out
timeout 2400 python -m pytest tests -m gpu -q -x > gpurun_out/r2_pytest3.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_pytest3.log
V64="a1=256.1.1.2,rec=64.1.1,bptt=128.1.1,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0,pf=2,hov=0"
for f in 0 3; do
  ASTRA_VARIANT="${V64/fwd=0/fwd=$f}" timeout 300 python bench.py --profile --steps 5 --batch 64 >> gpurun_out/r2_prof3.log 2>&1
done
V512="a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0"
ASTRA_VARIANT="$V512" timeout 300 python bench.py --profile --steps 5 >> gpurun_out/r2_prof3.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/r2_bench3.log 2>&1
