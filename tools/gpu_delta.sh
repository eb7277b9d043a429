#!/bin/bash
# Delta-pass check: parity suite, per-sweep trace, then the bench with and without it (LV_MOD_DELTA=0).
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > gpurun_out/delta_pytest.log 2>&1; echo "rc=$?" >> gpurun_out/delta_pytest.log
LV_TRACE=1 timeout 300 python tools/trace_run.py 27 > /dev/null 2> gpurun_out/delta_trace.err
timeout 600 python bench.py > gpurun_out/delta_bench_on.jsonl 2> gpurun_out/delta_bench_on.err
LV_MOD_DELTA=0 timeout 600 python bench.py > gpurun_out/delta_bench_off.jsonl 2> gpurun_out/delta_bench_off.err
timeout 900 python -m pytest tests/test_gpu_fullsize.py -x -q > gpurun_out/delta_pytest_full.log 2>&1; echo "rc=$?" >> gpurun_out/delta_pytest_full.log
