#!/bin/bash
mkdir -p gpurun_out
V="a1=256.1.1,rec=64.1.1,bptt=64.1.1,du=256.1.1,dw=256.1.1,dx=256.1.1,head=256.1.1,hdy=256.1.1,wg_side=1,bwd=0,pf=0,hov=0"
for i in 1 2; do for f in 0 1; do CFG_VARIANT="$V,fwd=$f" timeout 600 python scratch/cfg_bench.py cfg4 >> gpurun_out/r2_cfg52.jsonl 2>&1; done; done
