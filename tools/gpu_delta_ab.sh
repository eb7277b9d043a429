#!/bin/bash
# Delta-pass gate A/B: per-sweep modularity times of a full C5 run for several LV_DELTA_DIV values.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
for d in "$@"; do
  LV_DELTA_DIV=$d LV_TRACE=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/delta_div_$d.err
done
