#!/bin/bash
# Delta-pass gate on the other configs: LV_DELTA_DIV 1 (always) vs 1000000 (never) per config.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
for c in C2 C3 C4a C4b; do
  for d in 1 1000000; do
    LV_DELTA_DIV=$d timeout 600 python tools/run_time.py $c >> gpurun_out/delta_cfgs.jsonl 2>> gpurun_out/delta_cfgs.err
  done
done
