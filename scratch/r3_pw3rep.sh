#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_lm.py -m gpu -x -q -k "tiled" > gpurun_out/r3p3_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3p3_pytest.log
V64="a1=256.1.1.2,rec=64.1.1,bptt=64.1.1,du=224.1.1.2,dw=224.1.1.2,dx=224.1.1.2,head=128.1.1,hdy=128.1.1,wg_side=1,fwd=3,bwd=0,pf=2,hov=0,gc=3,wgs=1,bpw=2"
for r in 1 2 3; do
  ASTRA_VARIANT="$V64" timeout 300 python bench.py --batch 64 --no-tune --no-cpu-baseline --steps 20 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['regions_ms'], d['clocks'].get('sm_mhz'))" >> gpurun_out/r3p3_ab.log 2>&1
done
