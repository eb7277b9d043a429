#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
for pl in 8192 10240 12288; do
LV_PART_LABELS=$pl LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab15_$pl.err
done
