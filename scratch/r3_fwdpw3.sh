#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r3f3_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3f3_pytest.log
V="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0,gc=3,bpw=0"
for r in 1 2 3; do
  ASTRA_VARIANT="$V" timeout 300 python bench.py --no-tune --no-cpu-baseline --steps 20 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['regions_ms'], d['clocks'].get('sm_mhz'))" >> gpurun_out/r3f3_ab.log 2>&1
done
ASTRA_GRAPH=0 ASTRA_VARIANT="$V" timeout 600 ncu --set full --clock-control none -k regex:lstm_fwd_pw_kernel -s 150 -c 1 -o gpurun_out/r3f3_fwdpw python bench.py --profile --steps 1 > gpurun_out/r3f3_ncu.log 2>&1
python profiles/ncu_metrics.py gpurun_out/r3f3_fwdpw.ncu-rep > gpurun_out/r3f3_fwdpw_full.txt 2>&1
timeout 600 python scratch/cfg_bench.py cfg4 > gpurun_out/r3f3_cfg4.log 2>&1
