#!/bin/bash
mkdir -p gpurun_out
python bench.py > gpurun_out/r2s8_final_bench.log 2>&1
python bench.py --no-cpu-baseline > gpurun_out/r2s8_final_bench_rep2.log 2>&1
python bench.py --batch 64 --no-cpu-baseline > gpurun_out/r2s8_final_bench_b64.log 2>&1
V=$(grep '^{' gpurun_out/r2s8_final_bench.log | tail -1 | python -c "import json,sys; print(json.loads(sys.stdin.read())['tuner']['variant'])")
echo "$V" > gpurun_out/r2s8_final_variant.txt
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2s8_final_launches_cfg5_step.csv python bench.py --profile --steps 1 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2s8_final_launches_cfg5_step.csv > gpurun_out/r2s8_final_launches_summary.txt
