#!/bin/bash
mkdir -p gpurun_out
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_cfg2_launches.csv python scratch/prof_cfg2.py > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2_cfg2_launches.csv > gpurun_out/r2_cfg2_launches_summary.txt
