V="a1=256.1.1.2,rec=256.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=1"
TAG=${TAG:-bf1}
F="--set full --import-source on --clock-control none --cache-control none"
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" ncu $F -k regex:"bptt_fused" -s 50 -c 1 -o gpurun_out/${TAG} python bench.py --profile --steps 2 > gpurun_out/${TAG}.log 2>&1
ncu -i gpurun_out/${TAG}.ncu-rep --page details --csv > gpurun_out/${TAG}_details.csv 2>/dev/null
ncu -i gpurun_out/${TAG}.ncu-rep --page source --csv --print-source=sass > gpurun_out/${TAG}_sass.csv 2>/dev/null
