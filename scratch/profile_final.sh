# Round-1 final profile pass (run on the GPU box): bench line, launch list of one tuned cfg5 step,
# and ncu --set full captures of the dominant kernels.  Writes gpurun_out/fin_*.
set -x
python bench.py > gpurun_out/fin_bench.log 2>&1
V=$(tail -1 gpurun_out/fin_bench.log | python -c "import json,sys; print(json.loads(sys.stdin.read())['tuner']['variant'])")
echo "$V" > gpurun_out/fin_variant.txt
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/fin_launches_cfg5_step.csv python bench.py --profile --steps 1 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/fin_launches_cfg5_step.csv > gpurun_out/fin_launches_summary.txt
F="--set full --import-source on --clock-control none"
ncu $F -k regex:tc_gemm -s 2 -c 1 -o gpurun_out/fin_a1_gemm python scratch/gemm_one.py 51200 8192 2048 256 2 > /dev/null 2>&1
ncu $F -k regex:tc_gemm -s 2 -c 1 -o gpurun_out/fin_rec_gemm python scratch/gemm_one.py 512 8192 2048 256 2 > /dev/null 2>&1
ncu $F -k regex:tc_gemm -s 2 -c 1 -o gpurun_out/fin_bptt_gemm python scratch/gemm_one.py 512 2048 8192 256 2 1 1 4 > /dev/null 2>&1
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu $F --cache-control none -k regex:"lstm_fwd_pw" -s 250 -c 1 -o gpurun_out/fin_fwdpw python bench.py --profile --steps 2 > /dev/null 2>&1
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu $F --cache-control none -k regex:"lstm_bwd_pw" -s 150 -c 1 -o gpurun_out/fin_bwdpw python bench.py --profile --steps 2 > /dev/null 2>&1
for r in a1_gemm rec_gemm bptt_gemm fwdpw bwdpw; do python profiles/ncu_metrics.py gpurun_out/fin_$r.ncu-rep > gpurun_out/fin_${r}_full.txt 2>&1; done
ls -la gpurun_out/ | grep fin_
