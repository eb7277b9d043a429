#!/bin/bash
# One check call: GPU test suite, bench line, per-class trace of a full C5 run.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_check.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_check.log
timeout 600 python bench.py > gpurun_out/bench_check.jsonl 2> gpurun_out/bench_check.err
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/trace_check.err
