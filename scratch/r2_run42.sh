#!/bin/bash
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('SMOKE OK')" > gpurun_out/r2_smoke42.log 2>&1
echo "rc=$?" >> gpurun_out/r2_smoke42.log
timeout 1500 python -m pytest tests/ -m gpu -q > gpurun_out/r2_t42.log 2>&1
echo "rc=$?" >> gpurun_out/r2_t42.log
timeout 600 python bench.py > gpurun_out/r2_b42_default.log 2>&1
echo "rc=$?" >> gpurun_out/r2_b42_default.log
timeout 600 python bench.py --impl reference > gpurun_out/r2_b42_ref.log 2>&1
echo "rc=$?" >> gpurun_out/r2_b42_ref.log
