#!/bin/bash
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2s6_cfg4_launches.csv python scratch/prof_cfg4.py "a1=256.1.1.2,rec=64.1.1,bptt=64.1.1,du=256.1.1,dw=256.1.1,dx=256.1.1,head=256.1.1,hdy=256.1.1,wg_side=0,fwd=0,bwd=0,pf=0,hov=0" > gpurun_out/r2s6_cfg4_prof.log 2>&1
python profiles/summarise_launches.py gpurun_out/r2s6_cfg4_launches.csv > gpurun_out/r2s6_cfg4_launches_summary.txt
