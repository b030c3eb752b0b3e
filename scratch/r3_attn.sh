#!/bin/bash
# Fused attentive-decoder step: bitwise tests, then cfg4 A/B of fwd modes 0..3 and a tuned run.
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py -m gpu -x -q -k "attn" > gpurun_out/r3a_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3a_pytest.log
V="a1=256.1.1,rec=64.1.1,bptt=64.1.1,du=256.1.1,dw=256.1.1,dx=256.1.1,head=256.1.1,hdy=256.1.1,wg_side=0,bwd=0,pf=0,hov=0"
for m in 0 1 2 3 0 1 2 3; do CFG_VARIANT="$V,fwd=$m" timeout 300 python scratch/cfg_bench.py cfg4 >> gpurun_out/r3a_cfg4_ab.log 2>&1; done
timeout 300 python scratch/cfg_bench.py cfg4 > gpurun_out/r3a_cfg4_tuned.log 2>&1
