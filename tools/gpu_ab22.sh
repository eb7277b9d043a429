#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab22.err
LV_STAGE_A=1 LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab22_a.err
