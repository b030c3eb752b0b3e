#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py -q -x -k "row_streams or stream_schedules" > gpurun_out/r2_t12.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t12.log
V512="a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0"
for v in "rsp=0" "rsp=1" "rsp=0" "rsp=1" "rsp=1,rec=128.1.1.2" "rsp=1,bptt=128.1.1.2"; do
  ASTRA_VARIANT="$V512,$v" timeout 300 python bench.py --profile --steps 5 >> gpurun_out/r2_prof12.log 2>&1
done
