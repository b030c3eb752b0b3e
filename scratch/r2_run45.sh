#!/bin/bash
mkdir -p gpurun_out
L=$PWD/paper_conf_asplos_sivathanucsz19_b200/lib
V512="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=224.1.1.2,dw=256.1.1.2,dx=224.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0,gc=3"
V64="a1=256.1.1.2,rec=64.1.1,bptt=128.1.1,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=128.1.1,hdy=128.1.1,wg_side=1,fwd=3,bwd=0,pf=2,hov=0,gc=3,wgs=1,bpw=1"
for i in 1 2; do
 for lib in head 493249c 0b015a4; do
  if [ $lib = head ]; then O=""; else O=$L/libastra_ab_$lib.so; fi
  ASTRA_LIB_OVERRIDE=$O ASTRA_VARIANT="$V512" timeout 300 python bench.py --steps 20 >> gpurun_out/r2_ab45_512_$lib.log 2>&1
  ASTRA_LIB_OVERRIDE=$O ASTRA_VARIANT="$V64" timeout 300 python bench.py --steps 50 --batch 64 >> gpurun_out/r2_ab45_64_$lib.log 2>&1
 done
done
