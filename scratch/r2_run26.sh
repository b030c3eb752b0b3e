#!/bin/bash
mkdir -p gpurun_out
V="a1=256.1.1,rec=64.1.1,bptt=64.1.1,du=256.1.1,dw=256.1.1,dx=256.1.1,head=256.1.1,hdy=256.1.1,wg_side=0,fwd=0,bwd=0,pf=0,hov=0"
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_cfg4_launches26.csv python scratch/prof_cfg4.py "$V" > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2_cfg4_launches26.csv > gpurun_out/r2_cfg4_launches26_summary.txt
