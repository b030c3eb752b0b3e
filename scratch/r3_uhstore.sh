#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py -m gpu -x -q -k "fused_forward or graph_replay or recompute or variants_bitwise or fwd" > gpurun_out/r3u_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3u_pytest.log
V="a1=256.1.1.2,rec=256.1.1,bptt=256.1.1.2,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,hdy=256.1.1,wg_side=1,bwd=0,pf=0,hov=0,gc=3,bpw=0"
for r in 1 2 3; do for f in 0 1; do
  echo "== fwd=$f" >> gpurun_out/r3u_ab.log
  ASTRA_VARIANT="$V,fwd=$f" timeout 300 python bench.py --no-tune --no-cpu-baseline --steps 20 2>&1 | grep '^{' | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['regions_ms'], d['clocks'].get('sm_mhz'))" >> gpurun_out/r3u_ab.log 2>&1
done; done
