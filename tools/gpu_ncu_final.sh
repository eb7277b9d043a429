#!/bin/bash
# ncu --set full of the top kernels of level-0 sweep 1 on C5 (final code of the round)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
P="python tools/prof_sweep.py --scale 27 --what sweep1"
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
timeout 600 $NCU -k regex:k_stage --launch-skip 2 --launch-count 1 -o gpurun_out/ncuF_stage_b7 $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_cta --launch-skip 1 --launch-count 1 -o gpurun_out/ncuF_cta_1024 $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_part_stream --launch-count 1 -o gpurun_out/ncuF_pstream $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_small --launch-count 1 -o gpurun_out/ncuF_small4 $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_warp_l --launch-count 1 -o gpurun_out/ncuF_warp_b6 $P > /dev/null 2>&1
for f in gpurun_out/ncuF_*.ncu-rep; do ncu -i $f --page details > ${f%.ncu-rep}.details.txt 2>&1; ncu -i $f --page source --csv --print-source sass > ${f%.ncu-rep}.sass.csv 2>/dev/null; done
