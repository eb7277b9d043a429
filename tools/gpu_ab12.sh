#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab12.err
LV_TRACE=2 LV_GTAB_AGG=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab12_agg.err
LV_TRACE=2 LV_STREAM_MAXP=100000 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab12_all.err
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_ab12.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_ab12.log
timeout 600 python bench.py > gpurun_out/bench12.jsonl 2> gpurun_out/bench12.err
