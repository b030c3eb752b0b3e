#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r3bp_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3bp_pytest.log
timeout 900 python scratch/cfg_bench.py > gpurun_out/r3bp_cfgs.log 2>&1
python bench.py --batch 64 --no-cpu-baseline > gpurun_out/r3bp_bench_b64.log 2>&1
V="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0,gc=3,bpw=0"
for r in 1 2 3; do
  ASTRA_VARIANT="$V" timeout 300 python bench.py --no-tune --no-cpu-baseline --steps 20 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['regions_ms'], d['clocks'].get('sm_mhz'))" >> gpurun_out/r3bp_ab.log 2>&1
done
