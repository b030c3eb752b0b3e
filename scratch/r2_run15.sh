#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_lm.py tests/test_gpu_trajectory.py tests/test_gpu_fullsize.py -q -x > gpurun_out/r2_t15.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t15.log
timeout 600 python scratch/cfg_bench.py cfg2 > gpurun_out/r2_cfg15.jsonl 2>&1
timeout 600 python scratch/cfg_bench.py cfg3 >> gpurun_out/r2_cfg15.jsonl 2>&1
timeout 300 python bench.py --steps 20 > gpurun_out/r2_b15_512.log 2>&1
timeout 300 python bench.py --steps 20 --batch 64 > gpurun_out/r2_b15_64.log 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_cfg2_launches15.csv python scratch/prof_cfg2.py > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2_cfg2_launches15.csv > gpurun_out/r2_cfg2_launches15_summary.txt
