#!/bin/bash
mkdir -p gpurun_out
V512="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=224.1.1.2,dw=256.1.1.2,dx=224.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0,gc=3"
for i in 1 2 3; do
  ASTRA_VARIANT="$V512" timeout 300 python bench.py --steps 20 >> gpurun_out/r2_ab44_new.log 2>&1
  ASTRA_LIB_OVERRIDE=$PWD/paper_conf_asplos_sivathanucsz19_b200/lib/libastra_ab.so ASTRA_VARIANT="$V512" timeout 300 python bench.py --steps 20 >> gpurun_out/r2_ab44_old.log 2>&1
done
