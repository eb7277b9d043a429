#!/bin/bash
# One change, measured: parity files, C5 bench (5 steps), serialised per-class trace.
cd "$GRAFT_REPO_ROOT"; mkdir -p gpurun_out; O=gpurun_out/${1:-ab}; mkdir -p $O
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x > $O/pytest.log 2>&1; echo "rc=$?" >> $O/pytest.log
B="python bench.py --steps 5 --warmup 3 --no-cpu-baseline --e2e-steps 1 --e2e-warmup 0"
timeout 600 $B > $O/bench.jsonl 2> $O/bench.err
timeout 600 $B --config C3 > $O/bench_C3.jsonl 2> $O/bench_C3.err
LV_TRACE=2 timeout 300 python tools/trace_run.py 27 > /dev/null 2> $O/trace.err
