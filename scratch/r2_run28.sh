#!/bin/bash
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_lm.py tests/test_gpu_fullsize.py tests/test_gpu_trajectory.py -q -x > gpurun_out/r2_t28.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t28.log
V=$(cat gpurun_out/r2q_variant.txt)
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2q2_launches_cfg5_step.csv python bench.py --profile --steps 1 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2q2_launches_cfg5_step.csv > gpurun_out/r2q2_launches_summary.txt
timeout 600 python scratch/cfg_bench.py cfg2 > gpurun_out/r2_cfg28.jsonl 2>&1
