#!/bin/bash
mkdir -p gpurun_out
timeout 400 python -m pytest tests/test_gpu_cell.py -q -x -k "persistent_bptt" > gpurun_out/r2_t23.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t23.log
O=gpurun_out/r2_pb_sweep23.jsonl
PB_VARIANT="bwd=0,bptt=128.1.1,bpw=1,fwd=3" timeout 120 python scratch/pb_sweep.py >> $O 2>&1
timeout 120 python scratch/pb_sweep.py >> $O 2>&1
SB_B=128 PB_VARIANT="bwd=0,bptt=128.1.1,bpw=1,fwd=3" timeout 120 python scratch/pb_sweep.py >> $O 2>&1
SB_B=128 timeout 120 python scratch/pb_sweep.py >> $O 2>&1
timeout 300 python bench.py --steps 20 --batch 64 > gpurun_out/r2_b23_64.log 2>&1
