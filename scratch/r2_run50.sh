#!/bin/bash
mkdir -p gpurun_out
L=$PWD/paper_conf_asplos_sivathanucsz19_b200/lib
V512="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=224.1.1.2,dw=256.1.1.2,dx=224.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0,gc=3"
V64="a1=256.1.1.2,rec=64.1.1,bptt=128.1.1,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=128.1.1,hdy=128.1.1,wg_side=1,fwd=3,bwd=0,pf=2,hov=0,gc=3,wgs=1"
timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "bwd_pointwise_forms" > gpurun_out/r2_t50.log 2>&1
ASTRA_LIB_OVERRIDE=$L/libastra_ab_ub64.so timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "bwd_pointwise_forms" >> gpurun_out/r2_t50.log 2>&1
for i in 1 2; do
 for o in "" "$L/libastra_ab_ub64.so"; do
  for bp in 0 1; do
   ASTRA_LIB_OVERRIDE=$o ASTRA_VARIANT="$V512,bpw=$bp" timeout 300 python bench.py --steps 20 --profile >> gpurun_out/r2_ab50_512_$(basename "${o:-head}")_$bp.log 2>&1
   ASTRA_LIB_OVERRIDE=$o ASTRA_VARIANT="$V64,bpw=$bp" timeout 300 python bench.py --steps 50 --batch 64 --profile >> gpurun_out/r2_ab50_64_$(basename "${o:-head}")_$bp.log 2>&1
  done
 done
done
