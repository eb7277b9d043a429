#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
P="python tools/prof_sweep.py --scale 27 --what sweep1"
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
timeout 900 $NCU -k regex:k_stage --launch-skip 2 --launch-count 1 -o gpurun_out/ncu_stage_b7 $P > gpurun_out/ncu_a.log 2>&1
timeout 900 $NCU -k regex:sweep_cta --launch-skip 1 --launch-count 1 -o gpurun_out/ncu_cta_b7s1 $P > gpurun_out/ncu_b.log 2>&1
timeout 900 $NCU -k regex:sweep_part --launch-count 1 -o gpurun_out/ncu_part_b7 $P > gpurun_out/ncu_c.log 2>&1
timeout 900 $NCU -k regex:sweep_small --launch-count 1 -o gpurun_out/ncu_small4 $P > gpurun_out/ncu_d.log 2>&1
