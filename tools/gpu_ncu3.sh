#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
P="python tools/prof_sweep.py --scale 27 --what sweep1"
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
timeout 600 $NCU -k regex:sweep_part_stream --launch-count 1 -o gpurun_out/ncu3_pstream $P > gpurun_out/ncu3_a.log 2>&1
timeout 600 $NCU -k regex:sweep_small --launch-count 1 -o gpurun_out/ncu3_small4 $P > gpurun_out/ncu3_b.log 2>&1
timeout 600 $NCU -k regex:k_stage --launch-skip 2 --launch-count 1 -o gpurun_out/ncu3_stage_b7 $P > gpurun_out/ncu3_c.log 2>&1
for f in gpurun_out/ncu3_*.ncu-rep; do ncu -i $f --page details > ${f%.ncu-rep}.details.txt 2>&1; ncu -i $f --page source --csv --print-source sass > ${f%.ncu-rep}.sass.csv 2>/dev/null; done
