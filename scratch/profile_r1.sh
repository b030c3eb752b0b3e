# round-1 profile pass (run on the GPU box): launch list of one cfg5 step + full captures
python bench.py --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/prof_bench.log 2>&1
V=$(tail -1 gpurun_out/prof_bench.log | python -c "import json,sys; print(json.loads(sys.stdin.read())['tuner']['variant'])")
echo "$V" > gpurun_out/prof_variant.txt
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/r1_launches_cfg5_step.csv python bench.py --profile --steps 1 > /dev/null 2>&1
F="--set full --import-source on --clock-control none"
ncu $F -k regex:tc_gemm -s 2 -c 1 -o gpurun_out/r1_a1_gemm python scratch/gemm_one.py 51200 8192 2048 256 2 > /dev/null 2>&1
ncu $F -k regex:tc_gemm -s 2 -c 1 -o gpurun_out/r1_rec_gemm python scratch/gemm_one.py 512 8192 2048 256 2 > /dev/null 2>&1
ncu $F -k regex:tc_gemm -s 2 -c 1 -o gpurun_out/r1_bptt_gemm python scratch/gemm_one.py 512 2048 8192 256 2 1 1 4 > /dev/null 2>&1
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu $F --cache-control none -k regex:"lstm_.wd_pw" -s 250 -c 2 -o gpurun_out/r1_pw python bench.py --profile --steps 2 > /dev/null 2>&1
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu $F --cache-control none -k regex:"lstm_bwd_pw" -s 150 -c 1 -o gpurun_out/r1_bwdpw python bench.py --profile --steps 2 > /dev/null 2>&1
ls gpurun_out/*.ncu-rep
