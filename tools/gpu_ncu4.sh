#!/bin/bash
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
P="python tools/prof_sweep.py --scale 27 --what run"
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
timeout 900 $NCU -k regex:k_scatter_copy --launch-skip 1 --launch-count 1 -o gpurun_out/ncu4_copy_l1 $P > gpurun_out/ncu4_a.log 2>&1
timeout 900 $NCU -k regex:k_merge_warp --launch-count 1 -o gpurun_out/ncu4_mwarp_l0 $P > gpurun_out/ncu4_b.log 2>&1
for f in gpurun_out/ncu4_*.ncu-rep; do ncu -i $f --page details > ${f%.ncu-rep}.details.txt 2>&1; ncu -i $f --page source --csv --print-source sass > ${f%.ncu-rep}.sass.csv 2>/dev/null; done
