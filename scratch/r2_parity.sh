#!/bin/bash
# the whole GPU suite without -x, every parity metric logged (element-wise parity calibration)
mkdir -p gpurun_out
export ASTRA_PARITY_LOG=$PWD/gpurun_out/r2_parity_metrics.jsonl
rm -f $ASTRA_PARITY_LOG
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/r2_pytest_all.log 2>&1
echo "pytest rc=$?" >> gpurun_out/r2_pytest_all.log
