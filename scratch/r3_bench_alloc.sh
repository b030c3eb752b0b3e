#!/bin/bash
mkdir -p gpurun_out
python bench.py > gpurun_out/r3b_bench.log 2>&1
python bench.py --batch 64 --no-cpu-baseline > gpurun_out/r3b_bench_b64.log 2>&1
V="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=224.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0"
for g in 0 1 0 1; do ASTRA_VARIANT="$V,gc=3,gb=$g" python bench.py --no-cpu-baseline --steps 20 >> gpurun_out/r3b_ab.log 2>&1; done
for g in 0 1; do ASTRA_VARIANT="$V,gc=2,gb=$g" python bench.py --no-cpu-baseline --steps 20 >> gpurun_out/r3b_ab.log 2>&1; done
