#!/bin/bash
# tests + per-class trace (+ optional bench)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > gpurun_out/trace.out 2> gpurun_out/trace.err
LV_TRACE=1 LV_CONTRACT=hash timeout 300 python tools/trace_run.py 27 > gpurun_out/trace_hash.out 2> gpurun_out/trace_hash.err
if [ "$1" = "bench" ]; then timeout 600 python bench.py > gpurun_out/bench.jsonl 2> gpurun_out/bench.err; fi
