#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=1 LV_CONTRACT=hash timeout 300 python tools/trace_run.py 27 > gpurun_out/trace_hash.out 2> gpurun_out/trace_hash.err
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
LV_CONTRACT=hash timeout 1200 python -m pytest tests -m gpu -x -q -k "run or contract or aggregate or fullsize" > gpurun_out/pytest_gpu_hash.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu_hash.log
