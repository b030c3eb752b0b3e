#!/bin/bash
# GPU suite (element-wise parity, non-blocking tuner), bench, and the B=64 launch list
mkdir -p gpurun_out
export ASTRA_PARITY_LOG=$PWD/gpurun_out/r2_parity_metrics2.jsonl
rm -f $ASTRA_PARITY_LOG
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/r2_pytest2.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_pytest2.log
unset ASTRA_PARITY_LOG
timeout 900 python bench.py --steps 20 --warmup 5 > gpurun_out/r2_bench2.log 2>&1
V64="a1=256.1.1.2,rec=64.1.1,bptt=128.1.1,du=256.1.1.2,dw=256.1.1.2,dx=256.1.1.2,head=256.1.1,wg_side=1,fwd=0,bwd=0,pf=2,hov=0"
ASTRA_VARIANT=$V64 timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 2000 --csv --log-file gpurun_out/r2_b64_launches.csv python bench.py --profile --steps 1 --batch 64 > gpurun_out/r2_b64_prof.log 2>&1
