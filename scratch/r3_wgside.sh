#!/bin/bash
mkdir -p gpurun_out
V="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,hdy=256.1.1,bwd=0,pf=0,hov=0,gc=3,bpw=0"
for r in 1 2; do for w in 0 1; do for f in 0 1; do
  echo "== wg_side=$w fwd=$f" >> gpurun_out/r3w_ab.log
  ASTRA_VARIANT="$V,wg_side=$w,fwd=$f" timeout 300 python bench.py --no-tune --no-cpu-baseline --steps 20 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['regions_ms'], d['clocks'].get('sm_mhz'))" >> gpurun_out/r3w_ab.log 2>&1
done; done; done
