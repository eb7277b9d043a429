#!/bin/bash
# ncu --set full of the contraction kernels inside a C5 louvain_run (level 0 copy / merges /
# label partitions, level 2 combiner), summaries under gpurun_out/$1.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/${1:-ncuc}; mkdir -p $O
P="python tools/prof_sweep.py --scale 27 --what run"
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
timeout 600 $NCU -k regex:k_scatter_copy --launch-count 1 -o $O/ncu_copy $P > /dev/null 2>&1
timeout 600 $NCU -k regex:k_bigp_merge --launch-count 1 -o $O/ncu_bigp_merge $P > /dev/null 2>&1
timeout 600 $NCU -k regex:k_bigp_pass --launch-count 2 -o $O/ncu_bigp_pass $P > /dev/null 2>&1
timeout 600 $NCU -k regex:k_merge_warp --launch-count 2 -o $O/ncu_merge_warp $P > /dev/null 2>&1
timeout 600 $NCU -k regex:k_merge_mid --launch-count 2 -o $O/ncu_merge_mid $P > /dev/null 2>&1
timeout 600 $NCU -k regex:k_big_combine --launch-count 1 -o $O/ncu_combine $P > /dev/null 2>&1
timeout 600 $NCU -k regex:k_compact --launch-count 1 -o $O/ncu_compact $P > /dev/null 2>&1
for f in $O/ncu_*.ncu-rep; do
  ncu -i $f --page details > ${f%.ncu-rep}.details.txt 2>&1
  ncu -i $f --page source --csv > ${f%.ncu-rep}.sass.csv 2>/dev/null
done
