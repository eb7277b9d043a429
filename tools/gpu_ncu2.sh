#!/bin/bash
# ncu --set full of the table kernels of level-0 sweep 1 on C5 (one launch each)
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
P="python tools/prof_sweep.py --scale 27 --what sweep1"
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
timeout 600 $NCU -k regex:sweep_cta --launch-skip 1 --launch-count 1 -o gpurun_out/ncu2_cta_sub2 $P > gpurun_out/ncu2_a.log 2>&1
timeout 600 $NCU -k regex:sweep_warp --launch-skip 1 --launch-count 1 -o gpurun_out/ncu2_warp_b6 $P > gpurun_out/ncu2_b.log 2>&1
timeout 600 $NCU -k regex:sweep_part --launch-count 1 -o gpurun_out/ncu2_part $P > gpurun_out/ncu2_c.log 2>&1
for f in gpurun_out/ncu2_*.ncu-rep; do ncu -i $f --page details > ${f%.ncu-rep}.details.txt 2>&1; done
