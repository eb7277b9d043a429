#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab18.err
timeout 1500 python -m pytest tests -m gpu -x -q -k "contract or aggregate or run or fullsize or alternative" > gpurun_out/pytest_ab18.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ab18.log
timeout 600 python bench.py > gpurun_out/bench18.jsonl 2> gpurun_out/bench18.err
