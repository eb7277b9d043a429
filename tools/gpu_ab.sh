#!/bin/bash
# A/B of path-selection variants: one LV_TRACE=2 per-class timeline of a full C5 run
# per variant (plus the default), then python tools/ab_summary.py gpurun_out/ab_*.err
#   gpurun -- 'bash tools/gpu_ab.sh "LV_STREAM_MAXP=32" "LV_PART_LABELS=8192 LV_CAP_F=12"'
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab_default.err
i=0
for v in "$@"; do
  i=$((i + 1))
  env $v LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab_$i.err
  echo "$i: $v" >> gpurun_out/ab_variants.txt
done
