#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py -q -x -k "small_batch_persistent" > gpurun_out/sb_test.log 2>&1
echo "rc=$?" >> gpurun_out/sb_test.log
V64="a1=256.1.1.2,rec=64.1.1,bptt=128.1.1,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0,pf=2,hov=0"
for f in 0 3; do
  ASTRA_VARIANT="${V64/fwd=0/fwd=$f}" timeout 300 python bench.py --profile --steps 5 --batch 64 >> gpurun_out/sb_prof.log 2>&1
done
timeout 600 python bench.py --steps 20 --warmup 5 --batch 64 --no-cpu-baseline > gpurun_out/sb_bench64.log 2>&1
