#!/bin/bash
mkdir -p gpurun_out
V="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0,gc=3"
ASTRA_GRAPH=0 ASTRA_VARIANT="$V,bpw=2" timeout 600 ncu --set full --clock-control none --import-source on -k regex:lstm_bwd_pw3 -s 150 -c 1 -o gpurun_out/r3t_pw3 python bench.py --profile --steps 1 > gpurun_out/r3t_ncu1.log 2>&1
ASTRA_GRAPH=0 ASTRA_VARIANT="$V,bpw=0" timeout 600 ncu --set full --clock-control none --import-source on -k regex:lstm_bwd_pw_kernel -s 150 -c 1 -o gpurun_out/r3t_pw0 python bench.py --profile --steps 1 > gpurun_out/r3t_ncu2.log 2>&1
python profiles/ncu_metrics.py gpurun_out/r3t_pw3.ncu-rep > gpurun_out/r3t_pw3_full.txt 2>&1
python profiles/ncu_metrics.py gpurun_out/r3t_pw0.ncu-rep > gpurun_out/r3t_pw0_full.txt 2>&1
