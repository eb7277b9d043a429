#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_ab14.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ab14.log
timeout 600 python bench.py > gpurun_out/bench14.jsonl 2> gpurun_out/bench14.err
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab14.err
