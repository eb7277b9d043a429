#!/bin/bash
# End-of-round evidence (delta pass build): GPU suite, bench + reference arm, launch lists, ncu full of the delta kernel
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/r3_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/r3_pytest.log
bash tools/gpu_round2.sh
NCU="ncu --set full --import-source on --clock-control none"
timeout 900 $NCU -k regex:k_mod_delta_thr --launch-count 1 -o gpurun_out/ncuF_delta_thr python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
timeout 900 $NCU -k regex:k_mod_delta_warp --launch-skip 2 --launch-count 1 -o gpurun_out/ncuF_delta_warp python bench.py --steps 1 --warmup 3 --no-cpu-baseline > /dev/null 2>&1
for f in gpurun_out/ncuF_delta*.ncu-rep; do ncu -i $f --page details > ${f%.ncu-rep}.details.txt 2>&1; done
