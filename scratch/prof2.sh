# launch list (warm cache) + full captures of the chain pointwise kernels of the tuned cfg5 variant
V="a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0"
TAG=${TAG:-r1b}
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --cache-control none --csv --log-file gpurun_out/launches_$TAG.csv python bench.py --profile --steps 1 > gpurun_out/p_$TAG.log 2>&1
python profiles/summarise_launches.py gpurun_out/launches_$TAG.csv > gpurun_out/launches_${TAG}_summary.txt
F="--set full --import-source on --clock-control none --cache-control none"
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu $F -k regex:"lstm_bwd_pw" -s 150 -c 1 -o gpurun_out/${TAG}_bwdpw python bench.py --profile --steps 2 > /dev/null 2>&1
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu $F -k regex:"lstm_fwd_pw" -s 250 -c 1 -o gpurun_out/${TAG}_fwdpw python bench.py --profile --steps 2 > /dev/null 2>&1
ls -la gpurun_out/
