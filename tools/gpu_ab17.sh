#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab17.err
LV_SMALL2=0 LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab17_0.err
timeout 1500 python -m pytest tests -m gpu -x -q -k "parity" > gpurun_out/pytest_ab17.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ab17.log
