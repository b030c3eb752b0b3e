#!/bin/bash
# row_streams A/B at cfg5 B=512: one chain vs two row-half chains, forward pointwise grid capped
mkdir -p gpurun_out
V="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0,gc=3"
V2="a1=256.1.1.2,rec=224.1.1.2,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,fwd=0,bwd=0,pf=0,hov=0,gc=3"
for r in 1 2; do
for v in "$V" "$V,rsp=1" "$V2,rsp=1"; do
  for cap in 0 80 148; do
    echo "== $v cap=$cap" >> gpurun_out/r3r_ab.log
    ASTRA_FWDPW_CTAS=$cap ASTRA_VARIANT="$v" python bench.py --no-tune --no-cpu-baseline --steps 20 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['regions_ms'], d['clocks'].get('sm_mhz'))" >> gpurun_out/r3r_ab.log 2>&1
  done
done
done
