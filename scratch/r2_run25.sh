#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_fullsize.py -q -x -k "attn or cfg4" > gpurun_out/r2_t25.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t25.log
timeout 600 python scratch/cfg_bench.py cfg4 > gpurun_out/r2_cfg4_bench25.jsonl 2>&1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2_cfg4_launches25.csv python scratch/prof_cfg4.py > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2_cfg4_launches25.csv > gpurun_out/r2_cfg4_launches25_summary.txt
