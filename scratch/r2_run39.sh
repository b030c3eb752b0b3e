#!/bin/bash
mkdir -p gpurun_out
O=gpurun_out/r2_pb_sweep39.jsonl
PB_VARIANT="bwd=0,bptt=128.1.1,bpw=1,fwd=3" timeout 120 python scratch/pb_sweep.py > $O 2>&1
PB_VARIANT="bwd=0,bptt=64.1.1,bpw=1,fwd=3" timeout 120 python scratch/pb_sweep.py >> $O 2>&1
timeout 120 python scratch/pb_sweep.py >> $O 2>&1
ASTRA_PB_KA=4 ASTRA_PB_SA=2 ASTRA_PB_KB=4 ASTRA_PB_SB=2 ASTRA_PB_RES=-1 timeout 120 python scratch/pb_sweep.py >> $O 2>&1
timeout 300 python scratch/trace_sbbwd.py > gpurun_out/r2_sbbwd_trace39.jsonl 2>&1
