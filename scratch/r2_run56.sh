#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -m pytest tests/test_gpu_cell.py -q -x -k "rhn_persistent_bptt" > gpurun_out/r2_t56.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t56.log
V="a1=256.1.1,rec=64.1.1,bptt=64.1.1,du=64.1.1,dw=64.1.1,dx=128.1.1,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=1,pf=0,hov=0"
for i in 1 2; do for b in 0 1; do CFG_VARIANT="$V,bwd=$b" timeout 600 python scratch/cfg_bench.py cfg3 >> gpurun_out/r2_cfg56.jsonl 2>&1; done; done
