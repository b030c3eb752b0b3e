#!/bin/bash
mkdir -p gpurun_out
V64="a1=256.1.1.2,rec=64.1.1,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=128.1.1,hdy=128.1.1,wg_side=1,fwd=3,bwd=0,pf=2,hov=0,gc=3,wgs=1,bpw=1"
for i in 1 2; do
 for b in 128.1.1 64.1.1 64.2.1 64.1.2; do
  ASTRA_VARIANT="$V64,bptt=$b" timeout 300 python bench.py --steps 50 --batch 64 >> gpurun_out/r2_ab46_$b.log 2>&1
 done
done
