#!/bin/bash
# Source-level ncu (SASS + stall samples) of the current build's sweep and level kernels in
# level-0 sweep 1 of C5 (tools/prof_sweep.py), for stall attribution with tools/sass_lines.py.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/${1:-ncusrc}; mkdir -p $O
P="python tools/prof_sweep.py --scale 27 --what sweepq"
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
cap() { timeout 600 $NCU -k regex:$2 --launch-skip $3 --launch-count 1 -o $O/ncu_$1 $P > /dev/null 2>&1;
        ncu -i $O/ncu_$1.ncu-rep --page source --csv > $O/ncu_$1.sass.csv 2>/dev/null;
        ncu -i $O/ncu_$1.ncu-rep --page details > $O/ncu_$1.details.txt 2>&1; rm -f $O/ncu_$1.ncu-rep; }
cap small3 sweep_small 4          # b3 (deg 9-16) register kernel
cap warpd sweep_warp_d 0
cap warpc sweep_warp_c 0
cap cta0 sweep_cta_c 0
cap cta2 sweep_cta_c 1
cap pstream sweep_part_stream 0
cap commit k_commit 0
cap deltaw k_mod_delta_warp 0
cap deltat k_mod_delta_thr 0
