#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=1 timeout 300 python tools/trace_run.py 27 > gpurun_out/trace1.out 2> gpurun_out/trace1.err
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > gpurun_out/trace2.out 2> gpurun_out/trace2.err
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_q.jsonl 2> gpurun_out/bench_q.err
