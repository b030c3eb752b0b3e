#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py -m gpu -x -q -k "pointwise" > gpurun_out/r3b1_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3b1_pytest.log
V64="a1=256.1.1.2,rec=64.1.1,bptt=64.1.1,du=224.1.1.2,dw=224.1.1.2,dx=224.1.1.2,head=128.1.1,hdy=128.1.1,wg_side=1,fwd=3,bwd=0,pf=2,hov=0,gc=3,wgs=1"
for r in 1 2; do for b in 2 3; do
  echo "== B64 bpw=$b" >> gpurun_out/r3b1_ab.log
  ASTRA_VARIANT="$V64,bpw=$b" timeout 300 python bench.py --batch 64 --no-tune --no-cpu-baseline --steps 20 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['regions_ms'], d['clocks'].get('sm_mhz'))" >> gpurun_out/r3b1_ab.log 2>&1
done; done
V128="a1=256.1.1.2,rec=64.1.1,bptt=64.1.1,du=224.1.1.2,dw=224.1.1.2,dx=224.1.1.2,head=128.1.1,hdy=128.1.1,wg_side=1,fwd=3,bwd=0,pf=0,hov=0,gc=3"
for b in 0 1 2 3; do
  echo "== B128 bpw=$b" >> gpurun_out/r3b1_ab.log
  ASTRA_VARIANT="$V128,bpw=$b" timeout 300 python bench.py --batch 128 --no-tune --no-cpu-baseline --steps 20 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['regions_ms'], d['clocks'].get('sm_mhz'))" >> gpurun_out/r3b1_ab.log 2>&1
done
ASTRA_GRAPH=0 ASTRA_VARIANT="$V64,bpw=3" timeout 600 ncu --set full --clock-control none -k regex:lstm_bwd_pw1 -s 150 -c 1 -o gpurun_out/r3b1_pw1 python bench.py --profile --steps 1 --batch 64 > gpurun_out/r3b1_ncu.log 2>&1
python profiles/ncu_metrics.py gpurun_out/r3b1_pw1.ncu-rep > gpurun_out/r3b1_pw1_full.txt 2>&1
