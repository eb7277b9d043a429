#!/bin/bash
# big-segment contraction: 64-bit single sort (default) vs batched 32-bit sorts; contraction parity tests
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab5_sort64.err
LV_TRACE=2 LV_BIG_SORT32=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab5_sort32.err
timeout 900 python -m pytest tests -m gpu -x -q -k "contract or aggregate or run or fullsize" > gpurun_out/pytest_ab5.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ab5.log
