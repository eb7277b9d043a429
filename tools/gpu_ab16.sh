#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
for f in 8 12 16; do
LV_CAP_F=$f LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab16_$f.err
done
