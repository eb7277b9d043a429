#!/bin/bash
# A/B of sweep kernel variants: per-class LV_TRACE=2 timelines of a full C5 run
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab_default.err
LV_TRACE=2 LV_STAGE_W=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab_stagew.err
LV_TRACE=2 LV_CTA_PIPE=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab_ctapipe.err
LV_TRACE=2 LV_STREAM_MAXP=0 LV_PART_AGG=0 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab_pre_noagg.err
LV_TRACE=2 LV_STREAM_MAXP=0 LV_PART_AGG=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab_pre_agg.err
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
