#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab2_default.err
LV_TRACE=2 LV_STREAM_MAXP=0 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab2_allpre.err
LV_TRACE=2 LV_STREAM_MAXP=0 LV_PART_AGG=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab2_allpre_agg.err
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_q.jsonl 2> gpurun_out/bench_q.err
