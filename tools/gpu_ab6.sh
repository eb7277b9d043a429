#!/bin/bash
# A/B: direct-gather warp kernels for buckets 5-6 (LV_DIRECT=1) vs stage + warp kernels
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
LV_DIRECT=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "sweeps_bit_exact or full_run_bit_exact or aggregate" > gpurun_out/ab6_pytest_direct.log 2>&1; echo "rc=$?" >> gpurun_out/ab6_pytest_direct.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
timeout 300 $B > gpurun_out/ab6_direct0.jsonl 2>&1
LV_DIRECT=1 timeout 300 $B > gpurun_out/ab6_direct1.jsonl 2>&1
for c in C2 C3 C4b; do
  timeout 300 $B --config $c > gpurun_out/ab6_${c}_direct0.jsonl 2>&1
  LV_DIRECT=1 timeout 300 $B --config $c > gpurun_out/ab6_${c}_direct1.jsonl 2>&1
done
LV_DIRECT=1 LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab6_trace_direct.err
