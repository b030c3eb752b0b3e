V="a1=256.1.1,rec=64.1.1,bptt=64.1.1,du=64.1.1,dw=64.1.1,dx=256.1.1,head=256.1.1,wg_side=0,hov=0,fwd=1"
F="--set full --import-source on --clock-control none"
ASTRA_GRAPH=0 ncu $F -k regex:"rhn_rec_fwd" -c 1 -o gpurun_out/rhnf python scratch/prof_cfg3.py "$V" > gpurun_out/rhnf.log 2>&1
ncu -i gpurun_out/rhnf.ncu-rep --page details 2>/dev/null | grep -E "Duration|Throughput|Eligible|Active Warps|Stall|L2 Hit" | head -20
ncu -i gpurun_out/rhnf.ncu-rep --page source --csv --print-source sass 2>/dev/null > gpurun_out/rhnf_src.csv
