F="--set full --import-source on --clock-control none"
ncu $F -k regex:tc_gemm -s 2 -c 1 -o gpurun_out/r1_a1_gemm python scratch/gemm_one.py 51200 8192 2048 256 2 > /dev/null 2>&1
ncu $F -k regex:tc_gemm -s 2 -c 1 -o gpurun_out/r1_rec_gemm python scratch/gemm_one.py 512 8192 2048 256 2 > /dev/null 2>&1
ncu $F -k regex:tc_gemm -s 2 -c 1 -o gpurun_out/r1_bptt_gemm python scratch/gemm_one.py 512 2048 8192 256 2 1 1 4 > /dev/null 2>&1
ls gpurun_out/*.ncu-rep
