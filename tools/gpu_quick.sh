#!/bin/bash
# Quick check after a change: parity suites, one C5 bench line, per-class trace of a C5 run.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
T=${1:-q}
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q > gpurun_out/${T}_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/${T}_pytest.log
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0 > gpurun_out/${T}_bench.jsonl 2> gpurun_out/${T}_bench.err
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/${T}_trace.err
