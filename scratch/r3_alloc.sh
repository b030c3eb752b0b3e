#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_cell.py tests/test_gpu_lm.py -m gpu -q -k "gate_blocked or graph_replay or recompute_lm or fork_explores" > gpurun_out/r3g_pytest.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r3g_pytest.log
