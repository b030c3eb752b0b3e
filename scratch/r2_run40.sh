#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_gemm.py tests/test_gpu_cell.py -q -x -k "gemm or rhn or split" > gpurun_out/r2_t40.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t40.log
timeout 900 python -m pytest tests/test_gpu_gemm.py -q -x > gpurun_out/r2_t40b.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t40b.log
timeout 600 python scratch/cfg_bench.py cfg3 > gpurun_out/r2_cfg40.jsonl 2>&1
V512="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=224.1.1.2,dw=256.1.1.2,dx=224.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0,gc=3"
for v in "rec=256.1.1" "rec=224.1.1.2" "rec=256.1.1.2" "rec=128.1.1" "rec=256.1.1" "rec=224.1.1.2"; do
  ASTRA_VARIANT="$V512,$v" timeout 300 python bench.py --profile --steps 5 >> gpurun_out/r2_prof40.log 2>&1
done
