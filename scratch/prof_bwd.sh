V="a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0"
TAG=${TAG:-bwd2}
F="--set full --import-source on --clock-control none --cache-control none"
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu $F -k regex:"lstm_bwd_pw" -s 150 -c 1 -o gpurun_out/${TAG}_bwdpw python bench.py --profile --steps 2 > gpurun_out/${TAG}.log 2>&1
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none -k regex:"lstm_bwd_pw|tc_gemm" --csv --log-file gpurun_out/${TAG}_list.csv python bench.py --profile --steps 1 > /dev/null 2>&1
python profiles/summarise_launches.py gpurun_out/${TAG}_list.csv | head -5
