#!/bin/bash
# A/B: bucketised claim tables (LV_B4) and sweep graphs (LV_GRAPHS); parity of the defaults
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -k "not sampled_decisions" > gpurun_out/ab7_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/ab7_pytest.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
timeout 300 $B > gpurun_out/ab7_C5.jsonl 2>&1
LV_B4=0 timeout 300 $B > gpurun_out/ab7_C5_b4off.jsonl 2>&1
for c in C1 C2 C4a C4b; do
  timeout 300 $B --config $c --steps 10 > gpurun_out/ab7_$c.jsonl 2>&1
  LV_GRAPHS=0 timeout 300 $B --config $c --steps 10 > gpurun_out/ab7_${c}_graphs0.jsonl 2>&1
done
