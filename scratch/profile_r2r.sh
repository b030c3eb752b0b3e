#!/bin/bash
# Round-2 profile pass: bench lines + launch lists of one tuned step at B=512 and B=64, --set full
# captures of the round-2 kernels.  Writes gpurun_out/r2r_*.
mkdir -p gpurun_out
python bench.py > gpurun_out/r2r_bench.log 2>&1
V=$(tail -1 gpurun_out/r2r_bench.log | python -c "import json,sys; print(json.loads(sys.stdin.read())['tuner']['variant'])")
echo "$V" > gpurun_out/r2r_variant.txt
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2r_launches_cfg5_step.csv python bench.py --profile --steps 1 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2r_launches_cfg5_step.csv > gpurun_out/r2r_launches_summary.txt
python bench.py --batch 64 --no-cpu-baseline > gpurun_out/r2r_bench_b64.log 2>&1
V64=$(tail -1 gpurun_out/r2r_bench_b64.log | python -c "import json,sys; print(json.loads(sys.stdin.read())['tuner']['variant'])")
echo "$V64" > gpurun_out/r2r_variant_b64.txt
ASTRA_GRAPH=0 ASTRA_VARIANT="$V64" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2r_launches_b64_step.csv python bench.py --profile --steps 1 --batch 64 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2r_launches_b64_step.csv > gpurun_out/r2r_launches_b64_summary.txt
# --set full: the small-batch persistent forward, the wide backward pointwise (B=64), a1 (B=512)
ASTRA_GRAPH=0 ASTRA_VARIANT="$V64" timeout 900 ncu --set full --clock-control none --import-source on -k regex:lstm_fwd_persist -s 1 -c 1 -o gpurun_out/r2r_fwd_persist python bench.py --profile --steps 1 --batch 64 > gpurun_out/r2r_ncu1.log 2>&1
ASTRA_GRAPH=0 ASTRA_VARIANT="$V64" timeout 900 ncu --set full --clock-control none --import-source on -k regex:lstm_bwd_pw2 -s 150 -c 1 -o gpurun_out/r2r_bwd_pw2 python bench.py --profile --steps 1 --batch 64 > gpurun_out/r2r_ncu2.log 2>&1
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" timeout 900 ncu --set full --clock-control none --import-source on -k regex:tc_gemm2 -s 0 -c 1 -o gpurun_out/r2r_a1 python bench.py --profile --steps 1 > gpurun_out/r2r_ncu3.log 2>&1
for r in r2r_fwd_persist r2r_bwd_pw2 r2r_a1; do
  python profiles/ncu_metrics.py gpurun_out/$r.ncu-rep > gpurun_out/${r}_full.txt 2>&1
done
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r2r_cfg2_launches.csv python scratch/prof_cfg2.py > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/r2r_cfg2_launches.csv > gpurun_out/r2r_cfg2_launches_summary.txt
timeout 600 ncu --set full --clock-control none --import-source on -k regex:tc_gemm2 -s 4 -c 1 -o gpurun_out/r2r_cfg2_head python scratch/prof_cfg2.py > gpurun_out/r2r_ncu4.log 2>&1
python profiles/ncu_metrics.py gpurun_out/r2r_cfg2_head.ncu-rep > gpurun_out/r2r_cfg2_head_full.txt 2>&1
