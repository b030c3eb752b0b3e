#!/bin/bash
# Final pass: full GPU suite, smoke, bench lines (B=512 twice, B=64),
# launch lists of one tuned step, --set full of a1, the other configs, smoke().
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r2s7_pytest_all.txt 2>&1; echo "pytest rc=$?" >> gpurun_out/r2s7_pytest_all.txt
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2s7_smoke.txt 2>&1; echo "smoke rc=$?" >> gpurun_out/r2s7_smoke.txt
python bench.py > gpurun_out/r2s7_final_bench.log 2>&1
python bench.py --no-cpu-baseline > gpurun_out/r2s7_final_bench_rep2.log 2>&1
V=$(grep '^{' gpurun_out/r2s7_final_bench.log | tail -1 | python -c "import json,sys; print(json.loads(sys.stdin.read())['tuner']['variant'])")
echo "$V" > gpurun_out/r2s7_final_variant.txt
python bench.py --batch 64 --no-cpu-baseline > gpurun_out/r2s7_final_bench_b64.log 2>&1
V64=$(grep '^{' gpurun_out/r2s7_final_bench_b64.log | tail -1 | python -c "import json,sys; print(json.loads(sys.stdin.read())['tuner']['variant'])")
echo "$V64" > gpurun_out/r2s7_final_variant_b64.txt
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2s7_final_launches_cfg5_step.csv python bench.py --profile --steps 1 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2s7_final_launches_cfg5_step.csv > gpurun_out/r2s7_final_launches_summary.txt
ASTRA_GRAPH=0 ASTRA_VARIANT="$V64" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2s7_final_launches_b64_step.csv python bench.py --profile --steps 1 --batch 64 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2s7_final_launches_b64_step.csv > gpurun_out/r2s7_final_launches_b64_summary.txt
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" timeout 900 ncu --set full --clock-control none --import-source on -k regex:tc_gemm2 -s 0 -c 1 -o gpurun_out/r2s7_a1 python bench.py --profile --steps 1 > gpurun_out/r2s7_ncu_a1.log 2>&1
python profiles/ncu_metrics.py gpurun_out/r2s7_a1.ncu-rep > gpurun_out/r2s7_final_a1_full.txt 2>&1
timeout 900 python scratch/cfg_bench.py > gpurun_out/r2s7_cfgs.jsonl 2>&1
