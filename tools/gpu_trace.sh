#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > gpurun_out/trace.out 2> gpurun_out/trace.err
