#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > gpurun_out/smi.txt
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > gpurun_out/trace.out 2> gpurun_out/trace.err
timeout 600 python bench.py > gpurun_out/bench.jsonl 2> gpurun_out/bench.err
