#!/bin/bash
# A/B: register claim lists (default) vs table scans (LV_CLAIM=0); ncu of the degree-1 register kernel
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/ab3_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/ab3_pytest.log
LV_CLAIM=0 timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0 > gpurun_out/ab3_bench_claim0.jsonl 2>&1
timeout 300 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0 > gpurun_out/ab3_bench_claim1.jsonl 2>&1
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab3_trace.err
P="python tools/prof_sweep.py --scale 27 --what sweep1"
NCU="ncu --set full --import-source on --clock-control none --profile-from-start off"
timeout 600 $NCU -k regex:sweep_small --launch-count 1 -o gpurun_out/ab3_small1 $P > /dev/null 2>&1
timeout 600 $NCU -k regex:sweep_cta_c --launch-skip 1 --launch-count 1 -o gpurun_out/ab3_ctac $P > /dev/null 2>&1
for f in gpurun_out/ab3_*.ncu-rep; do
  ncu -i $f --page details > ${f%.ncu-rep}.details.txt 2>&1
  ncu -i $f --page source --csv > ${f%.ncu-rep}.sass.csv 2>/dev/null
done
