#!/bin/bash
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_cfg4_launches.csv python scratch/prof_cfg4.py > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2_cfg4_launches.csv > gpurun_out/r2_cfg4_launches_summary.txt
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_cfg3_launches.csv python scratch/prof_cfg3.py "a1=256.1.1,rec=64.1.1,bptt=64.1.1,du=64.1.1,dw=64.1.1,dx=128.1.1,head=256.1.1,wg_side=1,fwd=1,bwd=0,pf=0,hov=0" > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2_cfg3_launches.csv > gpurun_out/r2_cfg3_launches_summary.txt
timeout 600 python scratch/cfg_bench.py cfg4 > gpurun_out/r2_cfg4_bench.jsonl 2>&1
