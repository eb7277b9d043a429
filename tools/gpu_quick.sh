#!/bin/bash
# Quick check after a change: parity suites, then one bench line.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -x -q > gpurun_out/q_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/q_pytest.log
timeout 600 python bench.py > gpurun_out/q_bench.jsonl 2> gpurun_out/q_bench.err
