#!/bin/bash
# A/B of the 64-bit-key combiner of the contraction (LV_COMB64), parity suites
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q -k "not sampled_decisions" > gpurun_out/ab5_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/ab5_pytest.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
LV_COMB64=0 timeout 300 $B > gpurun_out/ab5_comb64_off.jsonl 2>&1
timeout 300 $B > gpurun_out/ab5_comb64_on.jsonl 2>&1
LV_TRACE=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/ab5_trace.err
