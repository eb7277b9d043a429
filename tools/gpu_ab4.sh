#!/bin/bash
# A/B of big-segment contraction variants (per-step LV_TRACE timelines of a full C5 run)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 LV_BIG_SORT64=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab4_sort64.err
LV_TRACE=2 LV_BIG_PART=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab4_part.err
